#!/bin/bash
# Round-2 job 8: GPU suite; sweep n = 33..64 at runtime chunks (RCW / RCW16 with
# 16-B cp.async staging, PTMEM) for the chunk 0 / 64 / 128 / other-chunk rows.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j8}; shift
WHAT=${*:-tests bench sweep}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
bench)
  t0=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - t0 ))s"
  tail -c 400 $O/bench.err ;;
sweep)
  timeout 1800 python scripts/autotune.py --n 33-64 --chunks 0,64,128,256 --reps 3 --variants 5,10,12 --out $O/sweep_33_64_rt.jsonl > $O/sweep.log 2>&1; echo "sweep rc=$?" ;;
esac; done
