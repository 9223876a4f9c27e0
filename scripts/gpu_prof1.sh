cd $GRAFT_REPO_ROOT
python scripts/prof_layer.py l2.3x3 3 > gpurun_out/prof1.txt 2>&1
ncu --set full --import-source on -k regex:k_tc_igemm -s 2 -c 1 -o gpurun_out/prof_l2_3x3 python scripts/prof_layer.py l2.3x3 3 >> gpurun_out/prof1.txt 2>&1
tail -3 gpurun_out/prof1.txt
