#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 EXTRA=-DALT_DBG_TILE=8 >/dev/null 2>&1
timeout 300 python scripts/exp_dbg4.py 2>&1 | grep -v "Exception ignored\|Traceback\|__del__\|AttributeError"
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
