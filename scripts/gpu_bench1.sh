cd $GRAFT_REPO_ROOT
timeout 300 python -m pytest tests/test_gpu_conv.py -q -k "tc_" 2>&1 | tail -3 > gpurun_out/tc2.txt
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
tail -3 gpurun_out/bench1.err
cat gpurun_out/tc2.txt
python -c "
import json; d=json.loads(open('gpurun_out/bench1.json').read().strip().splitlines()[-1])
for l in d.pop('per_layer'): print(l)
print(json.dumps(d, indent=1))
"
