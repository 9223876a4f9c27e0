#!/bin/bash
# re-tune (R50 layer set + chains) then the round evidence run
cd $GRAFT_REPO_ROOT
bash scripts/gpu_tune3.sh
bash scripts/gpu_r01_full.sh
