# final verification at HEAD: GPU suite, smoke, default bench line, reference arm
nvidia-smi --query-gpu=name,uuid,serial,driver_version,clocks.max.sm --format=csv > gpurun_out/box_id.txt 2>&1
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
