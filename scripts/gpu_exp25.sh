#!/bin/bash
for e in 11; do
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 EXTRA=-DALT_EXP=$e >/dev/null 2>&1
echo "== ALT_EXP=$e"
EPI_K=64 timeout 300 python scripts/exp_epi.py 2>&1
done
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
