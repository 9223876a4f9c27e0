#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -x -q -k "split or conv" 2>&1 | tail -3
timeout 120 python scripts/exp_dbg5.py l4.3x3 128 1 2 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
timeout 600 python scripts/exp_split.py l4.3x3,l4.3x3s2,l3.3x3,l4.1x1c,l2.1x1a 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
