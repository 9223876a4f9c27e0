python -m pytest tests/test_gpu_relayout.py tests/test_gpu_chain.py -q --timeout 900 -p no:cacheprovider > gpurun_out/t2.txt 2>&1; echo "rc=$?" >> gpurun_out/t2.txt
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_cases.py > gpurun_out/san_$tool.txt 2>&1; echo "rc=$?" >> gpurun_out/san_$tool.txt
done
python bench.py --steps 10 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
