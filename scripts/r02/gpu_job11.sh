#!/bin/bash
# Round-2 job 11: RCWP (paged TMEM, 2 CTAs/SM) -- RCW-family parity tests, sweep
# n = 33..64 (chunk 32 and 0) RCWP (param 0/1) vs RCW, ncu of RCWP at n = 64.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j11}; shift
WHAT=${*:-rtests sweep ncu}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
rtests)
  timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "rcw or bitwise or variants" > $O/pytest_rcw.log 2>&1; echo "rtests rc=$?"
  tail -n 3 $O/pytest_rcw.log ;;
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
sweep)
  timeout 1500 python scripts/autotune.py --n 33-64 --chunks 32,0 --reps 5 --variants 10,14 --out $O/sweep_rcwp.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
ncu)
  for d1 in 0 1; do
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf_rc --launch-skip 1 -c 1 -o $O/prof_rcwp64_d$d1 -f \
      python bench.py --workload c4n64 --batch 262144 --steps 1 --warmup 1 --per-n none --no-e2e --no-cpu-baseline \
      --tune "{\"variant\":14,\"threads_per_block\":256,\"param\":$d1,\"staging\":0}" > $O/ncu_d$d1.log 2>&1; echo "ncu d$d1 rc=$?"
  done ;;
ncuconv)
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:convert -c 8 -o $O/prof_conv -f \
    python scripts/r02/conv_probe.py 14 62 63 64 > $O/ncu_conv.log 2>&1; echo "ncuconv rc=$?" ;;
esac; done
python - "$O" <<'PY'
import json, sys
O = sys.argv[1]
try:
    rows = [json.loads(l) for l in open(f"{O}/sweep_rcwp.jsonl") if '"ms"' in l]
    for c in (32, 0):
        for n in range(33, 65):
            print(c, n, " ".join(f"v{r['variant']}p{r['param']}={r['gbs']:.0f}" for r in sorted([r for r in rows if r['n'] == n and r['chunk'] == c], key=lambda r: -r['gbs'])[:4]))
except Exception as e:
    print("sweep ERR", e)
PY
