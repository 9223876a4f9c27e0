#!/bin/bash
cd $GRAFT_REPO_ROOT; O=gpurun_out/prof_hbm; mkdir -p $O
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_relayout_row|k_dw|k_pool_vec8" -c 5 -o $O/hbm python scripts/prof_hbm_ops.py > $O/ncu.log 2>&1; echo rc=$?
tail -3 $O/ncu.log
python scripts/ncu_table.py $O/hbm.ncu-rep $O/table.txt
cat $O/table.txt
