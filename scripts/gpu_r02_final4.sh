# round-2 closing record at HEAD (after the bench pre-replay, fp32 full-size parity, store_at A4 assertion)
nvidia-smi --query-gpu=name,uuid,serial,driver_version,clocks.max.sm --format=csv > gpurun_out/box_id4.txt 2>&1
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider > gpurun_out/pytest_gpu4.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu4.txt
python __graft_entry__.py > gpurun_out/smoke4b.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke4b.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_final4.json 2> gpurun_out/bench_final4.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref4.json 2> gpurun_out/bench_ref4.err
