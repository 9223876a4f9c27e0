#!/bin/bash
cd $GRAFT_REPO_ROOT
for sk in 1 2; do timeout 120 python scripts/exp_dbg5.py l4.3x3 128 1 $sk 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"; done
timeout 120 python scripts/exp_dbg5.py l2.1x1a 128 1 2 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
