# ncu --set full of three representative R50 b32 layers at HEAD
for L in l1.3x3 l1.1x1b l4.1x1c l2.1x1a; do
  ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -s 4 -c 1 -o gpurun_out/s3_$L python scripts/one_layer.py $L 1 3 > gpurun_out/s3_$L.log 2>&1
done
python scripts/one_layer.py l1.3x3 1 3 > gpurun_out/s3_time.txt 2>&1
