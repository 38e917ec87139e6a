#!/bin/bash
# Round-2 job 9: GPU suite, bench, RCWD (diagonal warp) vs RCW at chunk 32, n = 49..64.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j9}; shift
WHAT=${*:-tests bench sweep}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 5 $O/pytest_gpu.log ;;
bench)
  t0=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - t0 ))s"
  tail -c 400 $O/bench.err ;;
sweep)
  timeout 900 python scripts/autotune.py --n 49-64 --chunks 32,0 --reps 5 --variants 10,12,13 --out $O/sweep_rcwd.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
esac; done
python - "$O" <<'PY'
import json, sys
O = sys.argv[1]
try:
    r = json.loads(open(f"{O}/bench.json").read().strip().splitlines()[-1])
    print("bench", r["value"], (r.get("roofline") or {}).get("frac"), (r.get("e2e") or {}).get("value"))
    for row in (r.get("per_n") or {}).get("rows", []):
        print("  n=%d v=%d %.4f %s" % (row["n"], row["variant"], row["frac"],
              {k: row[k] for k in ("convert_in_gbs", "convert_out_gbs") if k in row}))
    for row in (r.get("per_n_large_batch") or {}).get("rows", []):
        print("  L n=%d %.4f %s" % (row["n"], row["frac"], {k: row[k] for k in ("convert_in_gbs", "convert_out_gbs") if k in row}))
except Exception as e:
    print("bench ERR", e)
import collections
try:
    rows = [json.loads(l) for l in open(f"{O}/sweep_rcwd.jsonl") if '"ms"' in l]
    for c in (32, 0):
        print(c, " ".join(f"{n}:" + "/".join(f"{r['variant']}={r['gbs']:.0f}" for r in sorted([r for r in rows if r['n']==n and r['chunk']==c], key=lambda r: r['variant'])) for n in range(49, 65)))
except Exception as e:
    print("sweep ERR", e)
PY
