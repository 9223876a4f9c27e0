cd $GRAFT_REPO_ROOT
timeout 300 python scripts/exp_dbg.py 2>&1 | tail -30
