#!/bin/bash
# QTM sweep points for the tuning table: n = 33..64 at chunks 32, 0, 256.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 2400 python scripts/autotune.py --n 33-64 --chunks 32,0,256 --variants 8 --reps 3 --out gpurun_out/sweep_b200_r01j.jsonl > gpurun_out/sweep_j.log 2>&1
tail -2 gpurun_out/sweep_j.log; wc -l gpurun_out/sweep_b200_r01j.jsonl
