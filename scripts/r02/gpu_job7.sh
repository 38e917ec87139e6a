#!/bin/bash
# Round-2 job 7: GPU suite, smoke, default bench, reference arm, launch list and
# ncu --set full capture of the default (C3) kernel for roofline.traffic.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j7}; shift
WHAT=${*:-tests smoke bench ref launches ncu}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/smi.txt 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
smoke)
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
  tail -n 4 $O/smoke.log ;;
bench)
  t0=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - t0 ))s"
  tail -c 400 $O/bench.err ;;
ref)
  timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > $O/bench_ref.json 2> $O/bench_ref.err; echo "ref rc=$?" ;;
launches)
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv \
     python bench.py --steps 4 --warmup 3 --per-n none --no-e2e --no-cpu-baseline > $O/launches_bench.json 2>&1; echo "launches rc=$?" ;;
ncu)
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:potrf_ptmem --launch-skip 3 -c 1 \
     -o $O/prof_c3 -f python bench.py --steps 1 --warmup 3 --per-n none --no-e2e --no-cpu-baseline > $O/ncu_run.log 2>&1; echo "ncu rc=$?" ;;
esac; done
python - "$O" <<'PY'
import json, sys
O = sys.argv[1]
for f in ("bench", "bench_ref"):
    try:
        r = json.loads(open(f"{O}/{f}.json").read().strip().splitlines()[-1])
        print(f, r["value"], r["unit"], (r.get("roofline") or {}).get("frac"), (r.get("e2e") or {}).get("value"),
              (r.get("cpu_baseline") or {}).get("value"), r.get("clocks", {}) and r["clocks"].get("sm_mhz"))
        for row in (r.get("per_n") or {}).get("rows", []):
            print("  n=%d v=%d %.4f gbs=%.0f %s" % (row["n"], row["variant"], row["frac"], row["gbs"],
                  {k: row[k] for k in ("vs_copy", "convert_in_gbs", "convert_out_gbs") if k in row}))
        for row in (r.get("per_n_large_batch") or {}).get("rows", []):
            print("  L n=%d v=%d %.4f gbs=%.0f %s" % (row["n"], row["variant"], row["frac"], row["gbs"],
                  {k: row[k] for k in ("vs_copy", "convert_in_gbs", "convert_out_gbs") if k in row}))
    except Exception as e:
        print(f, "ERR", e)
PY
