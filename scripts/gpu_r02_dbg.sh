ISOLATED=1 python scripts/exp_dbg5.py l3.3x3,l2.3x3,l4.3x3 > gpurun_out/dbg_t0.txt 2>&1
ISOLATED=1 ALT_LIB_VARIANT=dbg3 python scripts/exp_dbg5.py l1.1x1b > gpurun_out/dbg_t3.txt 2>&1
