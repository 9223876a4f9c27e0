# A/B: one untimed replay of the K-step graph before the timed replay (graph upload + clock ramp) vs none
for i in 1 2; do
  for v in 0 1; do
    ALT_BENCH_PREREPLAY=$v python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/pr_r50_${v}_$i.json 2>/dev/null
    for w in mv2 bert r18; do ALT_BENCH_PREREPLAY=$v python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/pr_${w}_${v}_$i.json 2>/dev/null; done
  done
done
for f in gpurun_out/pr_*.json; do python -c "
import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['ms_per_step'], d['value'])"; done > gpurun_out/prereplay_ab.txt
