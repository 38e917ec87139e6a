#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python scripts/small_n_ceiling.py > gpurun_out/small_n.log 2>&1; tail -n 8 gpurun_out/small_n.log
