#!/bin/bash
# RCW at n = 25..32 (R = 4): parity at a few n, sweep chunk 32/0.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "bitwise and (25 or 29 or 31 or 32)" > gpurun_out/pytest_rcw32.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_rcw32.log
tail -n 2 gpurun_out/pytest_rcw32.log
timeout 900 python scripts/autotune.py --n 25-32 --chunks 32,0 --variants 10 --reps 3 --out gpurun_out/sweep_b200_r01p.jsonl > gpurun_out/sweep_p.log 2>&1
tail -n 1 gpurun_out/sweep_p.log
