#!/bin/bash
# Round-1 evidence run: GPU tests, smoke, bench (default + other workloads), ncu launch list + one --set full capture.
cd $GRAFT_REPO_ROOT; O=gpurun_out/r01g; mkdir -p $O
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $O/smoke.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
for w in r18 mv2 bert relayout; do timeout 600 python bench.py --workload $w --no-cpu-baseline > $O/bench_$w.json 2>> $O/bench.err; echo "bench $w rc=$?"; done
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_ref.json 2>> $O/bench.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $O/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/launches_bench.log 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tc -c 23 \
  -o $O/r50_full python bench.py --steps 1 --warmup 0 --eager --no-cpu-baseline > $O/full.log 2>&1; echo "full rc=$?"
python scripts/ncu_table.py $O/r50_full.ncu-rep $O/r50_table.txt $O/traffic_r50.json | tail -5
tail -c 1500 $O/bench.json
