#!/bin/bash
# round-1 profiles: launch list of the bench command + one --set full capture of the 23 conv launches
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
mkdir -p gpurun_out/prof3
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/prof3/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/prof3/launches_bench.log 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -c 23 \
  -o gpurun_out/prof3/r50_full python bench.py --steps 1 --warmup 0 --eager --no-cpu-baseline > gpurun_out/prof3/full.log 2>&1
echo "full rc=$?"
python scripts/ncu_table.py gpurun_out/prof3/r50_full.ncu-rep gpurun_out/prof3/r50_table.txt gpurun_out/prof3/traffic_r50.json | tail -30
timeout 300 python bench.py --steps 20 --warmup 5 > gpurun_out/prof3/bench.json 2>gpurun_out/prof3/bench.err
tail -c 600 gpurun_out/prof3/bench.json
