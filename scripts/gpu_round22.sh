#!/bin/bash
# ncu full capture of QTM at n=64 (P=4, 512 cols) and n=48, source-level stalls.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf_qtm -s 1 -c 1 \
  -o gpurun_out/prof_qtm64 python bench.py --n 64 --batch 262144 --chunk 32 --kind dd \
  --tune '{"variant":8,"threads_per_block":128,"param":4,"staging":2}' --steps 1 --warmup 1 \
  --no-cpu-baseline --no-e2e > gpurun_out/ncu_qtm64.log 2>&1
tail -3 gpurun_out/ncu_qtm64.log
