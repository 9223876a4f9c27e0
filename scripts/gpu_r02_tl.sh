# on-device per-CTA timelines (first tile and 4th tile) of two R50 b32 layers
for L in l1.3x3 l1.1x1b l2.1x1a; do ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/tl0_$L.txt 2>&1; python scripts/exp_dbg5.py $L > gpurun_out/tl0b_$L.txt 2>&1; done
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean > /dev/null 2>&1; make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j16 EXTRA=-DALT_DBG_TILE=3 > gpurun_out/tl_build.txt 2>&1
for L in l1.3x3 l1.1x1b l2.1x1a; do ISOLATED=1 python scripts/exp_dbg5.py $L > gpurun_out/tl3_$L.txt 2>&1; done
