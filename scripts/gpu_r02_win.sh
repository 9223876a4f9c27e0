# K_WIN knob sweep on R3 (threads per CTA, staging budget, fp32)
for th in 512 1024; do for b in 110000 200000; do
ALT_WIN_FP32=1 ALT_WIN_THREADS=$th ALT_WIN_BUDGET=$b python scripts/relayout_probe.py R3 >> gpurun_out/win_sweep2.txt 2>&1
done; done
