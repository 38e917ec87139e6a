#!/bin/bash
# Round-2 job 18: compute-sanitizer memcheck / racecheck / synccheck on the
# round-2 kernels (CANON, conversion v3, RCWP runtime-chunk prefetch).
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j18}; shift
O=gpurun_out/$TAG; mkdir -p $O
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python scripts/r02/sanitize_probe.py > $O/san_$tool.log 2>&1; echo "$tool rc=$?"
  tail -n 3 $O/san_$tool.log
done
