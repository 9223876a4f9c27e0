#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/diag3.py 2>&1 | grep GEMM
ALT_PDL=0 timeout 300 python scripts/diag3.py 2>&1 | grep GEMM | sed 's/^/nopdl /'
