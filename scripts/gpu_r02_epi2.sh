# drain anatomy of l1.1x1b: timelines with round stores off / output stores skipped
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean > /dev/null 2>&1; make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j16 EXTRA=-DALT_DBG_TILE=3 > gpurun_out/tl_build.txt 2>&1
for L in l1.1x1b l1.3x3; do
ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/te_base_$L.txt 2>&1
ALT_TC_ROUND=0 ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/te_r0_$L.txt 2>&1
ALT_TC_EPI_DBG=1 ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/te_d1_$L.txt 2>&1
ALT_TC_EPI_DBG=2 ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/te_d2_$L.txt 2>&1
done
