# MN-major tensor-core parity, one process per case (a device fault stays in its case)
python -m pytest tests/test_gpu_mnmajor.py --collect-only -q 2>/dev/null | grep '::' > /tmp/ids.txt
: > gpurun_out/mn_each.txt
while read id; do
  timeout 120 python -m pytest "$id" -q -x --timeout 100 -p no:cacheprovider > /tmp/one.txt 2>&1
  echo "$? $id $(grep -E '^E ' /tmp/one.txt | head -2 | cut -c1-200 | tr '\n' ' ')" >> gpurun_out/mn_each.txt
done < /tmp/ids.txt
python -m pytest "tests/test_gpu_store_at.py::test_matmul_store_at_parity" -q -p no:cacheprovider > gpurun_out/sa.txt 2>&1
