python -c "
import sys, json, torch; sys.path.insert(0, '.')
import bench_workloads as BW
r = BW.relayout_run(10, 1, torch.device('cuda', 0))
print(json.dumps(r))" > gpurun_out/rl.json 2> gpurun_out/rl.err
ALT_RELAYOUT_NOCT=1 python -c "
import sys, json, torch; sys.path.insert(0, '.')
import bench_workloads as BW
r = BW.relayout_run(10, 1, torch.device('cuda', 0))
print(json.dumps(r))" > gpurun_out/rl_noct.json 2>> gpurun_out/rl.err
python -m pytest tests/test_gpu_relayout.py -q -x --timeout 900 -p no:cacheprovider > gpurun_out/t3.txt 2>&1; echo "rc=$?" >> gpurun_out/t3.txt
