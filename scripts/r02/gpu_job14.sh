#!/bin/bash
# Round-2 job 14: full GPU suite, smoke, default bench (C3 + per-n block with the
# RCWP table rows and conversion v3), ncu of conversion v3 (n = 63) vs v2 (n = 64).
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j14}; shift
WHAT=${*:-tests smoke bench ncuconv}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
tests)
  timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
smoke)
  timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -n 4 $O/smoke.log ;;
bench)
  t0=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall=$(( $(date +%s) - t0 ))s"
  tail -c 300 $O/bench.err ;;
ncuconv)
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:convert -c 4 -o $O/prof_conv -f \
    python scripts/r02/conv_probe.py 63 64 > $O/ncu_conv.log 2>&1; echo "ncuconv rc=$?" ;;
esac; done
