#!/bin/bash
# PTMEM variant: targeted parity first (fast fail), then the whole gpu suite, sweep of new points
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "bitwise_identical and (32 or 24 or 28)" > gpurun_out/pytest_ptmem.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ptmem.log
tail -5 gpurun_out/pytest_ptmem.log
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python scripts/autotune.py --n 24-32 --chunks 32,64,0 --variants 5 --out gpurun_out/sweep_c.jsonl > gpurun_out/sweep_c.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/sweep_c.log
