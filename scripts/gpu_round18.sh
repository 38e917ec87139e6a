#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_solve.py tests/test_gpu_layout_synth_host.py -q -x -p no:cacheprovider > gpurun_out/pytest_solve.log 2>&1; tail -n 15 gpurun_out/pytest_solve.log
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 10 python -m pytest tests/test_gpu_solve.py -q -p no:cacheprovider -k "bitwise" > gpurun_out/sanitizer_solve.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/sanitizer_solve.log; tail -n 3 gpurun_out/sanitizer_solve.log
timeout 900 python scripts/solve_bench.py > gpurun_out/solve_bench.log 2>&1; tail -n 20 gpurun_out/solve_bench.log
timeout 900 python scripts/c4_sweep.py --no-cusolver --n 1-32 > gpurun_out/c4.log 2>&1
python - <<'PY'
import json
for l in open('gpurun_out/c4.jsonl'):
    r=json.loads(l); print(r['n'], round(r['convert_gbs']), end='; ')
PY
