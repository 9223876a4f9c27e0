make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean > /dev/null 2>&1; make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j16 EXTRA=-DALT_DBG_TILE=3 > gpurun_out/tl_build.txt 2>&1
ISOLATED=1 python scripts/exp_dbg5.py l1.3x3 > gpurun_out/t3_h2d.txt 2>&1
ALT_TC_EPI_DBG=3 ISOLATED=1 python scripts/exp_dbg5.py l1.3x3 > gpurun_out/t3_h2d_d3.txt 2>&1
ALT_TC_EPI_DBG=2 ISOLATED=1 python scripts/exp_dbg5.py l1.3x3 > gpurun_out/t3_h2d_d2.txt 2>&1
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean > /dev/null 2>&1; make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j16 EXTRA=-DALT_DBG_TILE=0 > gpurun_out/tl_build.txt 2>&1
ISOLATED=1 python scripts/exp_dbg5.py l1.3x3 > gpurun_out/t0_h2d.txt 2>&1
