#!/bin/bash
# RCW (v2 kernel) sweep for the remaining chunk sizes (64, 128, 256) at n = 33..64.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1200 python scripts/autotune.py --n 33-64 --chunks 64,128,256 --variants 10 --reps 3 --out gpurun_out/sweep_b200_r01n.jsonl > gpurun_out/sweep_n.log 2>&1
tail -n 1 gpurun_out/sweep_n.log
