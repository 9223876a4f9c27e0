# evidence run: launch list + traffic of the R50 step, full GPU suite, smoke, default bench line
nvidia-smi --query-gpu=name,uuid,serial,driver_version,clocks.max.sm --format=csv > gpurun_out/box_id.txt 2>&1; hostname >> gpurun_out/box_id.txt
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum,lts__t_sectors_op_write.sum --clock-control none -k regex:k_tc_conv --csv --log-file gpurun_out/traffic_r50.csv python scripts/one_step_r50.py > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r50.csv python bench.py --steps 2 --warmup 1 --no-aux --no-cpu-baseline > /dev/null 2>&1
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
