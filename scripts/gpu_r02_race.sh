python scripts/repro_store_at2.py 30 > gpurun_out/race2_default.txt 2>&1
ALT_PDL=0 python scripts/repro_store_at2.py 30 > gpurun_out/race2_nopdl.txt 2>&1
