#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_solve.py -q -x -p no:cacheprovider > gpurun_out/pytest_solve.log 2>&1; tail -15 gpurun_out/pytest_solve.log
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python scripts/zerocopy_probe.py > gpurun_out/zerocopy.log 2>&1; tail -30 gpurun_out/zerocopy.log | cut -c1-220
timeout 900 python scripts/c4_sweep.py --no-cusolver --n 1-32 > gpurun_out/c4.log 2>&1
