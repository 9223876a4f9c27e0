# depthwise register budget sweep (ALT_DW_MINB = resident CTAs per SM): MV2 chain + parity
for mb in 2 3 4; do
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean > /dev/null 2>&1; make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j16 EXTRA=-DALT_DW_MINB=$mb > /dev/null 2>&1
cuobjdump -res-usage paper_conf_eurosys_xuxpwwwdxcwc23_b200/libalt.so 2>/dev/null | grep -A1 k_dw3x3_fast | tail -1 > gpurun_out/dw_res$mb.txt
python -m pytest tests/test_gpu_conv.py -q -x -p no:cacheprovider -k "dw or depthwise" >> gpurun_out/dw_res$mb.txt 2>&1
for r in 1 2; do python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/dw_mv2_$mb$r.json 2>/dev/null; done
done
