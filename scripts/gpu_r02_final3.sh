# round-2 closing evidence (after the randomized-stress fixes: Ho=1 stores, X0 settle, lossy oracle reads, halo + MN-major B, grouped k-tile offsets)
nvidia-smi --query-gpu=name,uuid,serial,driver_version,clocks.max.sm --format=csv > gpurun_out/box_id3.txt 2>&1
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider > gpurun_out/pytest_gpu3.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu3.txt
python __graft_entry__.py > gpurun_out/smoke3.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke3.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_final3.json 2> gpurun_out/bench_final3.err
for w in r18 mv2 bert relayout; do python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench3_$w.json 2>/dev/null; done
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref3.json 2> gpurun_out/bench_ref3.err
