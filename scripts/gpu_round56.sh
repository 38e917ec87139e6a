#!/bin/bash
# Fill the sweep gaps: PTMEM (cp.async) at chunks 128/256/512 for n = 24..44, RCW at 512 for n = 33..64.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1200 python scripts/autotune.py --n 24-44 --chunks 128,256,512 --variants 5 --reps 3 --out gpurun_out/sweep_b200_r01r.jsonl > gpurun_out/sweep_r.log 2>&1
tail -n 1 gpurun_out/sweep_r.log
timeout 900 python scripts/autotune.py --n 33-64 --chunks 512 --variants 10,12 --reps 3 --out gpurun_out/sweep_b200_r01s.jsonl > gpurun_out/sweep_s.log 2>&1
tail -n 1 gpurun_out/sweep_s.log
