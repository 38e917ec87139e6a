#!/bin/bash
# Round-2 job 23 (final pass): GPU suite, smoke, default bench (C3 + per-n incl.
# conversion v2/v3/v4 and the fused canonical column, n <= 8 also at 64M), C5 on
# one GPU (32M matrices), reference arm.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j23}; shift
WHAT=${*:-tests smoke bench c5 ref}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
smoke)
  timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -n 5 $O/smoke.log ;;
bench)
  t0=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - t0 ))s"
  tail -c 300 $O/bench.err ;;
c5)
  t0=$(date +%s); timeout 900 python bench.py --workload c5 --steps 5 --warmup 3 --per-n none > $O/bench_c5.json 2> $O/bench_c5.err; echo "c5 rc=$? wall=$(( $(date +%s) - t0 ))s"
  tail -c 300 $O/bench_c5.err ;;
ref)
  timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; echo "ref rc=$?"; tail -c 300 $O/bench_ref.json ;;
esac; done
