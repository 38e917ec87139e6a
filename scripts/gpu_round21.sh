#!/bin/bash
# QTM (P threads per matrix, on-chip) first GPU pass: parity + sweep n = 33..64.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "qtm" > gpurun_out/pytest_qtm.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_qtm.log
tail -n 15 gpurun_out/pytest_qtm.log
timeout 1200 python scripts/autotune.py --n 33-64 --chunks 32 --variants 8 --reps 3 --out gpurun_out/sweep_qtm.jsonl > gpurun_out/sweep_qtm.log 2>&1
python - <<'PY'
import json, collections
best = collections.defaultdict(dict)
for l in open('gpurun_out/sweep_qtm.jsonl'):
    r = json.loads(l)
    if 'gbs' not in r: continue
    k = (r['variant'], r['param'], r['staging'], r['threads_per_block'])
    v = best[r['n']]
    if r['variant'] not in v or v[r['variant']][0] < r['gbs']:
        v[r['variant']] = (r['gbs'], k)
for n in sorted(best):
    print(n, {k: v for k, v in best[n].items()})
PY
