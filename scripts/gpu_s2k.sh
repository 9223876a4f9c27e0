#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 60 ./scripts/micro/tmem_bw2 2>&1 | tee gpurun_out/s2k_tmem2.txt
