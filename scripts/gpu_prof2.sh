cd $GRAFT_REPO_ROOT
for L in l1.1x1b l4.3x3 conv1; do
ncu --set full --import-source on -k regex:k_tc_conv -s 3 -c 1 -o gpurun_out/prof_$L python scripts/prof_layer.py $L 3 > gpurun_out/prof_$L.txt 2>&1
done
ls gpurun_out
