cd $GRAFT_REPO_ROOT
timeout 300 python scripts/exp_dbg2.py 2>&1 | grep -v "Exception\|Traceback\|destroy\|line 1"
