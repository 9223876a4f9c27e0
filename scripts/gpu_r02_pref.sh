# weight L2 prefetch before the PDL wait: parity smoke + A/B
python -m pytest tests/test_gpu_conv.py tests/test_gpu_conv3d.py -q -x -p no:cacheprovider --timeout 900 > gpurun_out/pref_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/pref_pytest.txt
for r in 1 2; do
for v in 0 1; do
if [ $v = 1 ]; then export ALT_TC_NO_BPREF=1; else unset ALT_TC_NO_BPREF; fi
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/r50_pref$v$r.json 2> /dev/null
python bench.py --batch 1 --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/r50b1_pref$v$r.json 2> /dev/null
python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r18_pref$v$r.json 2> /dev/null
python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/mv2_pref$v$r.json 2> /dev/null
python bench.py --workload bert --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bert_pref$v$r.json 2> /dev/null
done; done
