cd $GRAFT_REPO_ROOT
timeout 300 python -m pytest tests/test_gpu_relayout.py -q -x 2>&1 | tail -4
timeout 300 python scripts/exp_relayout.py 2>&1 | tail -30
