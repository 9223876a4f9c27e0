#!/bin/bash
cd $GRAFT_REPO_ROOT
for env in "X=1" "ALT_PDL=0" "ALT_PDL_CC=0" "ALT_PDL=0 ALT_PDL_CC=0"; do
  echo "== $env"; env $env timeout 600 python -m pytest tests/test_gpu_fullsize.py -x -q -k "resnet18 or mobilenet" 2>&1 | grep -E "passed|failed|AssertionError" | head -3
done
