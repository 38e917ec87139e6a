#!/bin/bash
# RCW (variant 10) sweep n = 33..64 (chunk 32, 0), and one bench run to see why it failed.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 200 python bench.py --n 64 --batch 1048576 --chunk 32 --tune '{"variant":10,"threads_per_block":256,"param":1,"staging":0}' --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b64.json 2> gpurun_out/b64.err
tail -c 600 gpurun_out/b64.json; tail -n 5 gpurun_out/b64.err
timeout 1200 python scripts/autotune.py --n 33-64 --chunks 32,0 --variants 10 --reps 3 --out gpurun_out/sweep_b200_r01l.jsonl > gpurun_out/sweep_l.log 2>&1
tail -n 2 gpurun_out/sweep_l.log
