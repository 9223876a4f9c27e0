#!/bin/bash
# same-box A/B of the R50 bench line: round-1 tree (.r01) vs the current tree
nvidia-smi --query-gpu=uuid,driver_version --format=csv,noheader > gpurun_out/ab_box.txt
for i in 1 2; do
  (cd .r01 && python bench.py --steps 20 --warmup 5 --no-cpu-baseline > ../gpurun_out/ab_r01_$i.json 2> ../gpurun_out/ab_r01_$i.err)
  python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-aux > gpurun_out/ab_cur_$i.json 2> gpurun_out/ab_cur_$i.err
done
