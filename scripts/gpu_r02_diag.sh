set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python scripts/exp_dbg5.py l1.1x1a,l1.1x1c,l4.1x1c,l3.1x1b,l2.3x3,l1.3x3 > gpurun_out/dbg_r50.txt 2>&1
ISOLATED=1 python scripts/exp_dbg5.py l1.1x1a,l4.1x1c > gpurun_out/dbg_r50_iso.txt 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench0.json 2> gpurun_out/bench0.err
