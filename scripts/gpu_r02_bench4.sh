# bench lines after the untimed graph pre-replay (graph upload no longer inside the timed region)
python bench.py --steps 10 --warmup 3 > gpurun_out/bench4.json 2> gpurun_out/bench4.err
ALT_BENCH_PREREPLAY=0 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench4_noprereplay.json 2>/dev/null
for w in r18 mv2 bert relayout; do python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench4_$w.json 2>/dev/null; done
python __graft_entry__.py > gpurun_out/smoke4.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke4.txt
