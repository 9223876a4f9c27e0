#!/bin/bash
cd $GRAFT_REPO_ROOT
for n in 32 256; do timeout 300 python scripts/exp_conv1.py $n 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"; done
