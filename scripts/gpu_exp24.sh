#!/bin/bash
for e in 5 6; do
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 EXTRA=-DALT_EXP=$e >/dev/null 2>&1
echo "== ALT_EXP=$e"
timeout 300 python scripts/exp_epi.py 2>&1 | grep "tiles/cta=32" | grep "K=64"
done
