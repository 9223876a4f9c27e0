#!/bin/bash
# extra bench workloads at N=1
set -x
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200/csrc -j8 >/dev/null 2>&1
mkdir -p gpurun_out
for w in r18 mv2 bert relayout; do
  timeout 300 python bench.py --workload $w --steps 10 --warmup 3 2>&1 | tail -3 | tee gpurun_out/wl_$w.json
done
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | tail -2
