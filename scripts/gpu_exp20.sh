#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 python scripts/exp_epi.py 2>&1
