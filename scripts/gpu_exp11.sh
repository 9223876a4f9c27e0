cd $GRAFT_REPO_ROOT
timeout 300 python -m pytest tests/test_gpu_conv.py -q -x -k "tc_" 2>&1 | tail -15
timeout 200 python scripts/exp_kscale.py 2>&1 | grep "stages=4" | tail -12
timeout 300 python -m pytest tests -q -x -m gpu 2>&1 | tail -3
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench11.json 2> gpurun_out/bench11.err
tail -2 gpurun_out/bench11.err
python -c "
import json; d=json.loads(open('gpurun_out/bench11.json').read().strip().splitlines()[-1])
for l in d.pop('per_layer'): print(l)
print({k: d[k] for k in ('value','ms_per_step','gpu_launches','e2e','clocks')}, d['roofline']['achieved'])
"
