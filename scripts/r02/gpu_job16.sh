#!/bin/bash
# Round-2 job 16: fused canonical factorization (batch_spotrf_canonical) --
# parity tests, ABI tests, and a short bench with the per-n block n = 1..24
# (fused canonical column for n <= 20) next to the interleaved kernel and the
# unfused canonical path.
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j16}; shift
WHAT=${*:-ctests pern}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
for w in $WHAT; do case $w in
ctests)
  timeout 1200 python -m pytest tests/test_gpu_canonical.py tests/test_abi.py -q -p no:cacheprovider -x > $O/pytest_canon.log 2>&1; echo "ctests rc=$?"
  tail -n 5 $O/pytest_canon.log ;;
pern)
  timeout 900 python bench.py --workload c2 --steps 3 --warmup 3 --per-n 1-24 --no-e2e --no-cpu-baseline > $O/bench_pern.json 2> $O/bench_pern.err; echo "pern rc=$?"
  tail -c 400 $O/bench_pern.err
  python scripts/per_n_table.py $O/bench_pern.json > $O/per_n.md; sed -n 5,32p $O/per_n.md ;;
ab)
  timeout 900 python scripts/r02/canon_ab.py > $O/canon_ab.jsonl 2> $O/canon_ab.err; echo "ab rc=$?"; tail -2 $O/canon_ab.err ;;
ncu)
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf_canon -c 2 -o $O/prof_canon -f \
    python scripts/r02/canon_probe.py 16 11 > $O/ncu.log 2>&1; echo "ncu rc=$?" ;;
esac; done
