for m in 0 1 2; do ALT_TC_EPI_DBG=$m python scripts/epi_probe.py > gpurun_out/epi_$m.txt 2>&1; done
