# LSU round stores: parity (conv/chain/fullsize) + A/B on the bench workloads
python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 1500 > gpurun_out/lsu_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/lsu_pytest.txt
for v in 1 0; do
ALT_TC_LSU=$v python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/r50_lsu$v.json 2> gpurun_out/r50_lsu$v.err
ALT_TC_LSU=$v python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r18_lsu$v.json 2> gpurun_out/r18_lsu$v.err
ALT_TC_LSU=$v python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/mv2_lsu$v.json 2> gpurun_out/mv2_lsu$v.err
ALT_TC_LSU=$v python bench.py --workload bert --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bert_lsu$v.json 2> gpurun_out/bert_lsu$v.err
done
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/r50_lsu1b.json 2> gpurun_out/r50_lsu1b.err
