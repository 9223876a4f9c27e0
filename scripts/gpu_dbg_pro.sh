#!/bin/bash
cd $GRAFT_REPO_ROOT
for L in l4.1x1b l1.1x1a; do
ISOLATED=1 timeout 120 python scripts/exp_dbg5.py $L 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
done
timeout 120 python scripts/exp_dbg5.py l4.1x1b 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
