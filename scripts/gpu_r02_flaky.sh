python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider -k "b1_tuned or parity" > gpurun_out/fl_e.txt 2>&1
python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider -k "bert or parity" > gpurun_out/fl_f.txt 2>&1
ALT_TC_ROUND=0 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider -k "bert or parity" > gpurun_out/fl_g.txt 2>&1
