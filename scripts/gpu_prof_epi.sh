#!/bin/bash
cd $GRAFT_REPO_ROOT; O=gpurun_out/prof_epi; mkdir -p $O
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -s 2 -c 1 -o $O/epi python scripts/prof_epi.py > $O/ncu.log 2>&1; echo rc=$?
