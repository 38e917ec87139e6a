#!/bin/bash
# REGV (variant 11): parity, then sweep n = 1..8 over chunks 32, 0, 256.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "regv or bitwise" > gpurun_out/pytest_regv.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_regv.log
tail -n 3 gpurun_out/pytest_regv.log
timeout 900 python scripts/autotune.py --n 1-8 --chunks 32,0,256 --variants 11 --reps 5 --out gpurun_out/sweep_b200_r01o.jsonl > gpurun_out/sweep_o.log 2>&1
tail -n 1 gpurun_out/sweep_o.log
