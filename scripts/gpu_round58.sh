#!/bin/bash
# Remaining sweep gaps: PTMEM chunk 64 (n=33-44); REGX/REGV chunks 64/128/512 (n<=16/8); RCW16 chunks 64/128/256.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python scripts/autotune.py --n 33-44 --chunks 64 --variants 5 --reps 3 --out gpurun_out/sweep_b200_r01t.jsonl > gpurun_out/sweep_t.log 2>&1
timeout 900 python scripts/autotune.py --n 1-16 --chunks 64,128,512 --variants 9,11 --reps 3 --out gpurun_out/sweep_b200_r01t.jsonl >> gpurun_out/sweep_t.log 2>&1
timeout 900 python scripts/autotune.py --n 49-64 --chunks 64,128,256 --variants 12 --reps 3 --out gpurun_out/sweep_b200_r01t.jsonl >> gpurun_out/sweep_t.log 2>&1
tail -n 1 gpurun_out/sweep_t.log; wc -l gpurun_out/sweep_b200_r01t.jsonl
