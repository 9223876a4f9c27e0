#!/bin/bash
cd $GRAFT_REPO_ROOT
for m in 0 1 2; do echo "== EPI_DBG=$m"; ALT_TC_EPI_DBG=$m timeout 300 python scripts/diag4.py 2>&1 | grep "^N="; done
