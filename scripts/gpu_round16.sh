#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python scripts/convert_sanity.py > gpurun_out/convert_plain.log 2>&1; tail -8 gpurun_out/convert_plain.log
timeout 900 compute-sanitizer --tool memcheck --print-limit 6 python scripts/convert_sanity.py > gpurun_out/convert_memcheck.log 2>&1; grep -E "ERROR SUMMARY|n [0-9]|ok|Invalid|Access|allocation" gpurun_out/convert_memcheck.log | head -30
timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "bitwise" > gpurun_out/pytest_bitwise.log 2>&1; tail -2 gpurun_out/pytest_bitwise.log
timeout 900 python scripts/autotune.py --n 4-20 --chunks 32 --variants 7 --out gpurun_out/sweep_i.jsonl > gpurun_out/sweep_i.log 2>&1
python - <<'PY'
import json
rows=[json.loads(l) for l in open('gpurun_out/sweep_i.jsonl')]
for r in rows: print(r['n'], r['param'], r.get('gbs'), r.get('error'))
PY
