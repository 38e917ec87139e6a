#!/bin/bash
# PANEL variant + REG occupancy: parity, sweep of the new points, ncu of n=32 winner
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 1200 python scripts/autotune.py --n 11-32 --chunks 32,64,128,256,512,0 --skip-from tuning/sweep_b200_r01a.jsonl --out gpurun_out/sweep_b.jsonl > gpurun_out/sweep_b.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/sweep_b.log
