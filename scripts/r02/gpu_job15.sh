#!/bin/bash
# Round-2 job 15: RCWP runtime-chunk prefetch with running pointers -- RCW-family
# parity tests and the chunk 0 / 64 sweep of RCWP at n = 49..64 (vs j11 / j12).
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j15}; shift
WHAT=${*:-rtests sweep}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
rtests)
  timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "rcw or bitwise or variants" > $O/pytest_rcw.log 2>&1; echo "rtests rc=$?"
  tail -n 2 $O/pytest_rcw.log ;;
sweep)
  timeout 1500 python scripts/autotune.py --n 49-64 --chunks 0,64 --reps 5 --variants 14 --out $O/sweep.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
esac; done
