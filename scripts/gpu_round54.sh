#!/bin/bash
# RCW16 (16 warps per 32 matrices): parity, then sweep n = 33..64 chunk 32 (and 0).
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "rcw or bitwise" > gpurun_out/pytest_rcw16.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_rcw16.log
tail -n 2 gpurun_out/pytest_rcw16.log
timeout 900 python scripts/autotune.py --n 33-64 --chunks 32,0 --variants 12 --reps 3 --out gpurun_out/sweep_b200_r01q.jsonl > gpurun_out/sweep_q.log 2>&1
tail -n 1 gpurun_out/sweep_q.log
