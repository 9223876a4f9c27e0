#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 120 ./scripts/micro/tma_bw 2>&1 | tee gpurun_out/s2f_tma.txt
