#!/bin/bash
# Round-2 job 10 (re-entry): GPU suite, default bench, RCWD vs RCW sweep at
# n = 49..64, ncu captures (with source) of RCW at n = 48 (2 CTAs/SM) and 64
# and of RCWD at n = 64.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j10}; shift
WHAT=${*:-tests bench sweep ncu}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
smoke)
  timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -n 4 $O/smoke.log ;;
bench)
  t0=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - t0 ))s"
  tail -c 300 $O/bench.err ;;
sweep)
  timeout 900 python scripts/autotune.py --n 45-64 --chunks 32 --reps 5 --variants 10,12,13 --out $O/sweep_rcwd.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
ncu)
  for tg in n48 n64 n64d; do
    nn=${tg:1:2}; TU=(); [ "$tg" = n64d ] && TU=(--tune '{"variant":13,"threads_per_block":288,"param":1,"staging":0}')
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf_rc --launch-skip 1 -c 1 -o $O/prof_rcw_$tg -f \
      python bench.py --workload c4n$nn --batch 262144 --steps 1 --warmup 1 --per-n none --no-e2e --no-cpu-baseline "${TU[@]}" > $O/ncu_$tg.log 2>&1; echo "ncu $tg rc=$?"
  done ;;
esac; done
python - "$O" <<'PY'
import json, sys
O = sys.argv[1]
try:
    r = json.loads(open(f"{O}/bench.json").read().strip().splitlines()[-1])
    print("bench", r["value"], (r.get("roofline") or {}).get("frac"), (r.get("e2e") or {}).get("value"))
    for row in (r.get("per_n") or {}).get("rows", []):
        print("  n=%d v=%d %.4f" % (row["n"], row["variant"], row["frac"]), {k: row[k] for k in ("convert_in_gbs", "convert_out_gbs") if k in row})
    for row in (r.get("per_n_large_batch") or {}).get("rows", []):
        print("  L n=%d %.4f" % (row["n"], row["frac"]))
except Exception as e:
    print("bench ERR", e)
try:
    rows = [json.loads(l) for l in open(f"{O}/sweep_rcwd.jsonl") if '"ms"' in l]
    for n in range(45, 65):
        print(n, " ".join(f"v{r['variant']}p{r['param']}={r['gbs']:.0f}" for r in sorted([r for r in rows if r['n'] == n], key=lambda r: -r['gbs'])[:4]))
except Exception as e:
    print("sweep ERR", e)
PY
