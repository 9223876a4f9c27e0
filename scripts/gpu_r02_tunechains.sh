mkdir -p gpurun_out/chains
python scripts/tune_chain_layouts.py gpurun_out/chains > gpurun_out/chains/log_all.txt 2>&1
