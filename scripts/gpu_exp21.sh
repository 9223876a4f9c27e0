#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 EXTRA=-DALT_DBG_TILE=4 >/dev/null 2>&1
timeout 300 python scripts/exp_dbg3.py 2>&1
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
