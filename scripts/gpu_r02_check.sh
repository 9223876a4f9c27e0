# round-2 check: full GPU suite, then the default bench line, then the 2-GPU spawn path
set -x
python -m pytest tests -m gpu -x -q --timeout 1500 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
python bench.py --gpus 2 --steps 3 --warmup 3 --no-aux > gpurun_out/bench_g2.json 2> gpurun_out/bench_g2.err; echo "g2 rc=$?" >> gpurun_out/bench_g2.err
