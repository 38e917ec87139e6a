#!/bin/bash
# Full GPU suite with QTM + new conversion; C4 n-sweep (factor, conversion, cuSOLVER context).
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 4 gpurun_out/pytest_gpu.log
timeout 1800 python scripts/c4_sweep.py --out gpurun_out/c4_r24.jsonl --md gpurun_out/c4_r24.md > gpurun_out/c4.log 2>&1
tail -n 3 gpurun_out/c4.log
