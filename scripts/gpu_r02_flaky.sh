python -m pytest tests/test_gpu_relayout.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider -k "parity or d6_set" > gpurun_out/fl_a.txt 2>&1
python -m pytest tests/test_gpu_mnmajor.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider > gpurun_out/fl_b.txt 2>&1
python -m pytest tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider > gpurun_out/fl_c.txt 2>&1
python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider -k "b1 or bert or parity" > gpurun_out/fl_d.txt 2>&1
bash scripts/gpu_r02_c3d.sh
