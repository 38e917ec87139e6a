#!/bin/bash
# Round-2 job 22: ncu captures of the PTMEM table kernels at n = 25 / 26 / 27
# (odd n below 0.85 of HBM) for a side-by-side.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j22}; shift
O=gpurun_out/$TAG; mkdir -p $O
for nn in 25 26 27; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf_ --launch-skip 1 -c 1 -o $O/prof_n$nn -f \
    python bench.py --workload c4n$nn --batch 1048576 --steps 1 --warmup 1 --per-n none --no-e2e --no-cpu-baseline > $O/ncu_n$nn.log 2>&1; echo "ncu n$nn rc=$?"
done
