cd $GRAFT_REPO_ROOT
timeout 300 python scripts/exp_tiles.py 2>&1 | tail -30
