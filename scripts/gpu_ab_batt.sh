#!/bin/bash
# A/B: libalt.so with and without the attached-bias epilogue read (ALT_NO_BATT), same box, alternating runs
cd paper_conf_eurosys_xuxpwwwdxcwc23_b200
make -s -j16 >/dev/null 2>&1 && cp libalt.so /tmp/alt_batt.so
make -s clean && make -s -j16 EXTRA=-DALT_NO_BATT >/dev/null 2>&1 && cp libalt.so /tmp/alt_nobatt.so
cd ..
for i in 1 2 3; do
  for v in batt nobatt; do
    cp /tmp/alt_$v.so paper_conf_eurosys_xuxpwwwdxcwc23_b200/libalt.so
    echo -n "$v "; timeout 300 python bench.py --no-cpu-baseline --steps 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['clocks']['sm_mhz'])"
  done
done
cp /tmp/alt_batt.so paper_conf_eurosys_xuxpwwwdxcwc23_b200/libalt.so
