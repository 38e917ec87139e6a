#!/bin/bash
# A/B of the 2-D TMA runtime-chunk staging (BSPOTRF_TMA2D=0 disables it): PTMEM
# (variant 5) and RCWP (14) at runtime chunks.
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/${1:-j27}; mkdir -p $O
for v in 1 0; do
  BSPOTRF_TMA2D=$v timeout 900 python scripts/autotune.py --n 24,25,28,32,33,36,40,44,48 --chunks 0,64 --reps 5 --variants 5,14 --out $O/sweep_tma$v.jsonl > $O/sweep_tma$v.log 2>&1; echo "tma$v rc=$?"
done
python - "$O" <<'PY'
import json, sys
O = sys.argv[1]
def best(f):
    d = {}
    for l in open(f):
        r = json.loads(l)
        if "gbs" in r:
            k = (r["n"], r["chunk"], r["variant"])
            d[k] = max(d.get(k, 0), r["gbs"])
    return d
a, b = best(f"{O}/sweep_tma1.jsonl"), best(f"{O}/sweep_tma0.jsonl")
for k in sorted(a):
    print(k, "tma2d", round(a[k]), "cp.async", round(b.get(k, 0)), f"{a[k] / b[k] - 1:+.1%}" if b.get(k) else "")
PY
