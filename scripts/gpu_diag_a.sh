#!/bin/bash
cd $GRAFT_REPO_ROOT; O=gpurun_out/diag_a; mkdir -p $O
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 300 python scripts/exp_dbg5.py l4.1x1b,l4.3x3,l1.1x1a,l2.1x1b > $O/dbg5.txt 2>&1; echo rc=$?
timeout 400 python scripts/diag1.py > $O/diag1.txt 2>&1; echo rc=$?
timeout 300 python scripts/chain_ops.py mv2 16 > $O/mv2_ops.txt 2>&1; timeout 300 python scripts/chain_ops.py r18 256 > $O/r18_ops.txt 2>&1
cat $O/dbg5.txt $O/diag1.txt $O/mv2_ops.txt $O/r18_ops.txt | head -250
