#!/bin/bash
# Round-2 job 13: conversion v3 (fixed slices, constant row phases) -- bitwise
# tests, A/B timing against v2 at n = 6..64 (1M, chunk 32); parity tests that
# go through the updated table (RCWP at n = 49..64).
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j13}; shift
WHAT=${*:-ctests ab}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
ctests)
  timeout 1200 python -m pytest tests/test_gpu_layout_synth_host.py -m gpu -q -p no:cacheprovider -x -k "conversion" > $O/pytest_conv.log 2>&1; echo "ctests rc=$?"
  tail -n 15 $O/pytest_conv.log ;;
ab)
  timeout 1200 python scripts/r02/conv_ab.py ${AB_N:-6-64} ${AB_P:-v2,v3} > $O/conv_ab.jsonl 2> $O/conv_ab.err; echo "ab rc=$?"; tail -3 $O/conv_ab.err ;;
ptests)
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "rcw or c4 or table or default" > $O/pytest_p.log 2>&1; echo "ptests rc=$?"
  tail -n 3 $O/pytest_p.log ;;
tests)
  timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log ;;
ncuconv)
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:convert -c 4 -o $O/prof_conv -f \
    python scripts/r02/conv_probe.py 63 62 > $O/ncu_conv.log 2>&1; echo "ncuconv rc=$?" ;;
esac; done
[ -f $O/conv_ab.jsonl ] && python - "$O" <<'PY'
import json, sys
rows = [json.loads(l) for l in open(f"{sys.argv[1]}/conv_ab.jsonl")]
by = {}
for r in rows: by.setdefault(r["n"], {})[r["path"]] = r
for n in sorted(by):
    print(n, " ".join(f"{p}: c {r['to_canon_frac']:.3f} i {r['to_inter_frac']:.3f}" for p, r in sorted(by[n].items())))
PY
