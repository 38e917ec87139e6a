#!/bin/bash
# Source-level ncu of RCW v4 at n=64 and n=56 (1 CTA/SM).
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for cfg in "64 1 w64"; do
  set -- $cfg
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf -s 1 -c 1 \
    -o gpurun_out/prof_$3 python bench.py --n $1 --batch 262144 --chunk 32 --tune "{\"variant\":10,\"threads_per_block\":256,\"param\":$2,\"staging\":0}" --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_$3.log 2>&1
  tail -n 1 gpurun_out/ncu_$3.log
done
