#!/bin/bash
# Round-2 job 12: RCWP vs RCW / RCW16 at the runtime chunks (64/128/256) for
# n = 45..64 -- the table rows the chunk-32/0 sweep of job 11 did not cover.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j12}; shift
O=gpurun_out/$TAG; mkdir -p $O
timeout 1500 python scripts/autotune.py --n 45-64 --chunks 64,128,256 --reps 5 --variants 10,12,14 --out $O/sweep_rcwp_rt.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?"
