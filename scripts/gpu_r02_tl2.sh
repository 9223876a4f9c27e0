# TMA-only cadence (ALT_TC_EPI_DBG=3: no MMA, no drain) of l1.3x3 / l1.1x1a, tile 3 timelines, and stage sweep
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean > /dev/null 2>&1; make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j16 EXTRA=-DALT_DBG_TILE=3 > gpurun_out/tl_build.txt 2>&1
for L in l1.3x3 l1.1x1a l2.3x3; do
ALT_TC_EPI_DBG=3 ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/tt_d3_$L.txt 2>&1
ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/tt_base_$L.txt 2>&1
done
python scripts/stage_probe.py l1.3x3,l2.3x3,l1.1x1a,l3.3x3 > gpurun_out/tt_stage_probe.txt 2>&1
ALT_TC_EPI_DBG=3 python scripts/stage_probe.py l1.3x3,l2.3x3,l1.1x1a,l3.3x3 > gpurun_out/tt_stage_probe_d3.txt 2>&1
