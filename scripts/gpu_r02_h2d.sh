# 2-D halo: parity, then A/B (ALT_TC_HROW=0) on the R50 set and the R18 chain
python -m pytest tests/test_gpu_conv.py -q -x -p no:cacheprovider -k "halo" > gpurun_out/h2d_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/h2d_pytest.txt
python scripts/one_layer.py l1.3x3 1 3 > gpurun_out/h2d_l13.txt 2>&1
ALT_TC_HROW=0 python scripts/one_layer.py l1.3x3 1 3 >> gpurun_out/h2d_l13.txt 2>&1
python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/h2d_r18_on.json 2>/dev/null
ALT_TC_HROW=0 python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/h2d_r18_off.json 2>/dev/null
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/h2d_r50_on.json 2>/dev/null
ALT_TC_HROW=0 python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/h2d_r50_off.json 2>/dev/null
