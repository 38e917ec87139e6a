#!/bin/bash
# Round-2 job 24: RCWP runtime-chunk staging by 2-D TMA -- RCW-family parity
# tests, then the runtime-chunk sweep of RCW / RCWP at n = 33..64.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j24}; shift
WHAT=${*:-rtests sweep}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
rtests)
  timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "rcw or bitwise or variants" > $O/pytest_rcw.log 2>&1; echo "rtests rc=$?"
  tail -n 2 $O/pytest_rcw.log ;;
sweep)
  timeout 1500 python scripts/autotune.py --n ${SW_N:-33-64} --chunks ${SW_C:-0,64,128,256} --reps 5 --variants ${SW_V:-10,14} --out $O/sweep.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
esac; done
