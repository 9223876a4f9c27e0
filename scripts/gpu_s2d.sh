#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python scripts/diag2.py 2>&1 | grep -v "^Exception ignored\|__del__\|AttributeError\|Traceback" | tee gpurun_out/s2d_diag2.txt
