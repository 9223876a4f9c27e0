# relayout kernels: parity + bench (new K_WIN / K_PBLOCK / warp-staged stores) and A/B knobs
python -m pytest tests/test_gpu_relayout.py -q -x -p no:cacheprovider > gpurun_out/rl_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/rl_pytest.txt
python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_new.json 2> gpurun_out/rl_new.err
ALT_RELAYOUT_NOWIN=1 ALT_RELAYOUT_NOPB=1 ALT_RELAYOUT_NOWS=1 python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_old.json 2> gpurun_out/rl_old.err
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv --log-file gpurun_out/rl_ncu.csv python bench.py --workload relayout --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
