#!/bin/bash
# Round-2 job 6: GPU suite, re-sweep n = 24..32 chunk 32 (FILL 12 for n <= 31), bench.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j6}; shift
WHAT=${*:-tests sweep bench}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
sweep)
  timeout 900 python scripts/autotune.py --n 24-32 --chunks 32 --reps 5 --variants 2,4,5 --out $O/sweep_24_32.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
bench)
  timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
  tail -c 600 $O/bench.err ;;
esac; done
python - "$O" <<'PY'
import json, sys
O = sys.argv[1]
try:
    r = json.loads(open(f"{O}/bench.json").read().strip().splitlines()[-1])
    print("bench", r["value"], r["unit"], (r.get("roofline") or {}).get("frac"), (r.get("e2e") or {}).get("value"),
          r.get("clocks", {}) and r["clocks"].get("sm_mhz"))
    for row in (r.get("per_n") or {}).get("rows", []):
        print("  n=%d v=%d %.4f gbs=%.0f %s" % (row["n"], row["variant"], row["frac"], row["gbs"],
              {k: row[k] for k in ("vs_copy", "convert_in_gbs", "convert_out_gbs") if k in row}))
    for row in (r.get("per_n_large_batch") or {}).get("rows", []):
        print("  L n=%d v=%d %.4f gbs=%.0f vs_copy=%s" % (row["n"], row["variant"], row["frac"], row["gbs"], row.get("vs_copy")))
except Exception as e:
    print("bench ERR", e)
PY
