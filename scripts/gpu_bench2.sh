cd $GRAFT_REPO_ROOT
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench2.json 2> gpurun_out/bench2.err
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --eager > gpurun_out/bench2e.json 2>> gpurun_out/bench2.err
tail -3 gpurun_out/bench2.err
for f in bench2 bench2e; do python -c "
import json; d=json.loads(open('gpurun_out/$f.json').read().strip().splitlines()[-1])
for l in d.pop('per_layer'): print(l)
print({k: d[k] for k in ('value','ms_per_step','gpu_launches','e2e','clocks')}, d['roofline']['achieved'])
"; done
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches2.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --eager > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/launches2.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
for r in rows[1:]:
    print(r[ki][:60], r[vi])
PY
