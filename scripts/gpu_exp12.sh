cd $GRAFT_REPO_ROOT
timeout 300 python scripts/exp_relayout.py 2>&1 | tail -30
