#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 EXTRA=-DALT_DBG_TILE=2 >/dev/null 2>&1
timeout 300 python scripts/exp_dbg5.py l1.3x3,l4.3x3,l1.1x1a 2>&1 | grep -v "Exception ignored\|Traceback\|__del__\|AttributeError" | tee gpurun_out/s2e.txt
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
