ALT_TC_EPI_DBG=3 python scripts/stage_probe.py l1.3x3,l3.3x3,l2.1x1a,l3.1x1a,l1.1x1a > gpurun_out/stages3.txt 2>&1
python scripts/stage_probe.py l1.3x3,l3.3x3,l2.1x1a,l3.1x1a,l1.1x1a > gpurun_out/stages0.txt 2>&1
