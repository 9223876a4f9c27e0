#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 600 python scripts/exp_split.py l4.3x3,l4.3x3s2,l3.3x3,l4.1x1c,l1.1x1b,l2.1x1a 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
