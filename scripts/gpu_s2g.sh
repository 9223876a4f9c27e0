#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 60 ./scripts/micro/op_lat 2>&1 | tee gpurun_out/s2g_oplat.txt
