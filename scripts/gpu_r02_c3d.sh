python -m pytest tests/test_gpu_conv3d.py --collect-only -q 2>/dev/null | grep '::' > /tmp/ids.txt
: > gpurun_out/c3d_each.txt
while read id; do
  timeout 300 python -m pytest "$id" -q -x --timeout 250 -p no:cacheprovider > /tmp/one.txt 2>&1
  echo "$? $id $(grep -E '^E ' /tmp/one.txt | head -2 | cut -c1-220 | tr '\n' ' ')" >> gpurun_out/c3d_each.txt
done < /tmp/ids.txt
