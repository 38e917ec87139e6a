#!/bin/bash
# Round-2 job 3: GPU suite, default bench (per-n), ncu captures of the
# conversion kernels (odd / even n) and of RCW at n = 64.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j5}; shift
WHAT=${*:-tests bench ncuconv}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
bench)
  timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
  tail -c 600 $O/bench.err ;;
ncuconv)
  timeout 900 ncu --set full --clock-control none -k regex:convert --launch-skip 0 -c 8 -o $O/prof_conv -f python scripts/r02/conv_probe.py 63 64 > $O/ncu_conv.log 2>&1; echo "ncuconv rc=$?" ;;
ncurcw)
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:potrf_rcw --launch-skip 1 -c 1 -o $O/prof_rcw64 -f \
     python bench.py --workload c4n64 --batch 262144 --steps 1 --warmup 1 --per-n none --no-e2e --no-cpu-baseline > $O/ncu_rcw.log 2>&1; echo "ncurcw rc=$?" ;;
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
