#!/bin/bash
# Source-level ncu of QTM at n=64 (streamed, 512 cols) and n=48 (preloaded), PTMEM at n=40.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for cfg in "64 262144 {\"variant\":8,\"param\":4,\"staging\":2} q64" "48 262144 {\"variant\":8,\"param\":4,\"staging\":3} q48" "40 262144 {\"variant\":5,\"threads_per_block\":128,\"param\":24,\"staging\":1} p40"; do
  set -- $cfg
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf -s 1 -c 1 \
    -o gpurun_out/prof_$4 python bench.py --n $1 --batch $2 --chunk 32 --tune "$3" --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_$4.log 2>&1
  tail -n 2 gpurun_out/ncu_$4.log
done
