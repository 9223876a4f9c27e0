# state check at HEAD: full GPU suite, smoke, default bench line, reference arm
nvidia-smi --query-gpu=name,uuid,clocks.max.sm --format=csv > gpurun_out/box_id.txt 2>&1
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider -x > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
