#!/bin/bash
# ncu evidence for the other configs: MV2 b16 chain, R18 b256 chain (one step each), relayout D6 set
cd $GRAFT_REPO_ROOT; O=gpurun_out/prof_chains; mkdir -p $O
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
cat > /tmp/one_chain.py <<'PY'
import sys, torch
sys.path.insert(0, ".")
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
ch = (CH.mobilenet_v2(16, torch.device("cuda", 0)) if sys.argv[1] == "mv2" else CH.resnet18(256, torch.device("cuda", 0)))
ch.run(); torch.cuda.synchronize()
import torch.cuda.profiler as prof
prof.start(); ch.run(); torch.cuda.synchronize(); prof.stop()
PY
for w in mv2 r18; do
  timeout 900 ncu --set full --clock-control none --profile-from-start off -o $O/$w python /tmp/one_chain.py $w > $O/$w.log 2>&1; echo "$w rc=$?"
  python scripts/ncu_table.py $O/$w.ncu-rep $O/${w}_table.txt > /dev/null 2>&1; tail -2 $O/${w}_table.txt; rm -f $O/$w.ncu-rep
done
cat > /tmp/relayout_set.py <<'PY'
import sys, torch
sys.path.insert(0, ".")
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import relayout_set
import torch.cuda.profiler as prof
dev = torch.device("cuda", 0)
items = []
for name, shape, sp, dp in relayout_set.cases():
    S, D = alt.Layout(shape, sp), alt.Layout(shape, dp)
    src = S.empty(torch.bfloat16, dev).normal_(); dst = D.empty(torch.bfloat16, dev)
    alt.relayout(S, src, D, dst); items.append((S, src, D, dst))
torch.cuda.synchronize()
prof.start()
for S, src, D, dst in items: alt.relayout(S, src, D, dst)
torch.cuda.synchronize(); prof.stop()
PY
timeout 900 ncu --set full --clock-control none --profile-from-start off -o $O/relayout python /tmp/relayout_set.py > $O/relayout.log 2>&1; echo "relayout rc=$?"
python scripts/ncu_table.py $O/relayout.ncu-rep $O/relayout_table.txt > /dev/null 2>&1; cat $O/relayout_table.txt; rm -f $O/relayout.ncu-rep
