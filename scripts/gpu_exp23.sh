#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_conv.py -q -x -k "config1 and NHWC" 2>&1 | grep -E "Error|error|assert|^E " | head -20
timeout 300 python scripts/exp_epi.py 2>&1 | tail -5
