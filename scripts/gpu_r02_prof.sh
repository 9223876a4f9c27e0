ncu --set full --clock-control none -k regex:k_tc_conv -s 6 -c 1 -o gpurun_out/prof_l13 python scripts/one_layer.py l1.3x3 1 3 > /dev/null 2>&1
ncu --set full --clock-control none -k regex:k_tc_conv -s 6 -c 1 -o gpurun_out/prof_l1b python scripts/one_layer.py l1.1x1b 1 3 > /dev/null 2>&1
