#!/bin/bash
# ncu of the conversion kernels at n=31 (32-bit canonical side) vs n=32 (128-bit).
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:convert -c 8 \
  -o gpurun_out/prof_convert python scripts/convert_probe.py 31,32 > gpurun_out/ncu_convert.log 2>&1
tail -2 gpurun_out/ncu_convert.log
