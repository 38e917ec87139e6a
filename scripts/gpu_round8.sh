#!/bin/bash
# PTMEM restructure: parity, PTMEM sweep, bench C3, ncu
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python scripts/autotune.py --n 24-32 --chunks 32,64,0 --variants 5 --out gpurun_out/sweep_f.jsonl > gpurun_out/sweep_f.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_ptmem32b python bench.py --workload c3 --steps 4 --warmup 3 --no-e2e --no-cpu-baseline --tune '{"variant":5,"threads_per_block":128,"param":16,"staging":1}' > gpurun_out/prof_ptmem32.out 2>&1
python - <<'PY'
import json
rows=[json.loads(l) for l in open('gpurun_out/sweep_f.jsonl')]
for n in range(24,33):
    rs=sorted([r for r in rows if r['n']==n and 'ms' in r], key=lambda r:r['ms'])[:2]
    print(n, [(r['chunk'], r['param'], r['staging'], r['gbs']) for r in rs])
print([r for r in rows if 'error' in r][:3])
PY
