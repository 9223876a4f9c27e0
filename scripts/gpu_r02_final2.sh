# round-2 final evidence (after the 2-D halo, re-tuned caches, depthwise register budget)
nvidia-smi --query-gpu=name,uuid,serial,driver_version,clocks.max.sm --format=csv > gpurun_out/box_id.txt 2>&1
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r50.csv python bench.py --steps 2 --warmup 1 --no-aux --no-cpu-baseline > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum,lts__t_sectors_op_write.sum --clock-control none -k regex:k_tc_conv --csv --log-file gpurun_out/traffic_r50.csv python scripts/one_step_r50.py > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -s 4 -c 1 -o gpurun_out/final_l13x3 python scripts/one_layer.py l1.3x3 1 3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -s 4 -c 1 -o gpurun_out/final_l41x1a python scripts/one_layer.py l4.1x1a 1 3 > /dev/null 2>&1
