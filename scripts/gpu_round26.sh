#!/bin/bash
# REGX (f3 axes) parity + sweep; ncu of the conversion kernels (n=31 vs 32).
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "regx or bitwise_identical" > gpurun_out/pytest_regx.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_regx.log
tail -n 3 gpurun_out/pytest_regx.log
timeout 1200 python scripts/autotune.py --n 1-16 --chunks 32,0,256 --variants 9 --reps 3 --out gpurun_out/sweep_b200_r01k.jsonl > gpurun_out/sweep_k.log 2>&1
tail -n 1 gpurun_out/sweep_k.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:convert -c 8 \
  -o gpurun_out/prof_convert python scripts/convert_probe.py 31,32 > gpurun_out/ncu_convert.log 2>&1
tail -n 1 gpurun_out/ncu_convert.log
