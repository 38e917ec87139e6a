#!/bin/bash
# Round-2 job 2: probes (FFMA2 rate, exhaustive fast sqrt/rcp), GPU suite,
# default bench, n<=4 sweep at 64M matrices, carveout sweep on table rows.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j2}; shift
WHAT=${*:-probes tests bench small carve}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
probes)
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include scripts/r02/ffma2_probe.cu -o /tmp/ffma2 && /tmp/ffma2 > $O/ffma2_probe.json 2>&1
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include scripts/r02/verify_fast_sqrt_rcp.cu -o /tmp/vfsr && timeout 300 /tmp/vfsr > $O/fast_sqrt_rcp.json 2>&1
  cat $O/ffma2_probe.json $O/fast_sqrt_rcp.json ;;
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
smoke)
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
  tail -n 2 $O/smoke.log ;;
bench)
  timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
  tail -c 600 $O/bench.err ;;
small)
  timeout 900 python scripts/autotune.py --n 1-4 --chunks 32,0 --batch 67108864 --reps 5 --variants 1,3,6,9,11 --out $O/sweep_small_64M.jsonl > $O/sweep_small.log 2>&1; echo "small rc=$?" ;;
carve)
  timeout 1200 python scripts/carveout_sweep.py --out $O/sweep_carveout.jsonl > $O/carve.log 2>&1; echo "carve rc=$?"; tail -3 $O/carve.log ;;
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
