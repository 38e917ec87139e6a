#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "bitwise or ragged or injected" > gpurun_out/pytest_par.log 2>&1; tail -2 gpurun_out/pytest_par.log
timeout 900 python scripts/autotune.py --n 24-32 --chunks 32 --variants 5 --out gpurun_out/sweep_g.jsonl > gpurun_out/sweep_g.log 2>&1
timeout 600 python scripts/probe_ceiling.py > gpurun_out/probe.log 2>&1; cat gpurun_out/probe.log
python - <<'PY'
import json
rows=[json.loads(l) for l in open('gpurun_out/sweep_g.jsonl')]
for n in range(24,33):
    rs=sorted([r for r in rows if r['n']==n and 'ms' in r], key=lambda r:r['ms'])[:2]
    print(n, [(r['param'], r['staging'], r['gbs']) for r in rs])
PY
