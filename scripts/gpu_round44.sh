#!/bin/bash
# A/B on one box: host copy pipeline with kernel copies vs DMA 2-D copies (C2, C3), twice each.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for rep in 1 2; do
for mode in kernel dma; do
  BSPOTRF_HOST_COPY=$mode timeout 600 python bench.py --no-cpu-baseline --steps 5 --warmup 3 --e2e-steps 3 > gpurun_out/ab_c2_$mode.json 2>/dev/null
  BSPOTRF_HOST_COPY=$mode timeout 900 python bench.py --workload c3 --no-cpu-baseline --steps 5 --warmup 3 --e2e-steps 3 > gpurun_out/ab_c3_$mode.json 2>/dev/null
  python - $mode <<'PY'
import json,sys
for f in ("gpurun_out/ab_c2_%s.json"%sys.argv[1],"gpurun_out/ab_c3_%s.json"%sys.argv[1]):
    r=json.loads(open(f).read().strip().splitlines()[-1]); e=r["e2e"]
    print(f, {k:(v["value"],v["ms_per_step"]) for k,v in e["paths"].items()})
PY
done
done
