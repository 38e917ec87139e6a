#!/bin/bash
# Round-2 job 26: PTMEM runtime-chunk staging by 2-D TMA -- full GPU suite, then
# the runtime-chunk sweep of PTMEM (and the table's alternatives) at n = 24..44.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j26}; shift
WHAT=${*:-tests sweep}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
sweep)
  timeout 1500 python scripts/autotune.py --n 24-44 --chunks 0,64,128,256 --reps 5 --variants 4,5,10,14 --out $O/sweep.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
esac; done
