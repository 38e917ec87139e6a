#!/bin/bash
# RTMA variant + PTMEM fix: targeted parity, whole suite, sweep of new points, ncu of RTMA n16 / PTMEM n32
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "bitwise_identical" > gpurun_out/pytest_bitwise.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_bitwise.log
tail -3 gpurun_out/pytest_bitwise.log
timeout 900 python scripts/autotune.py --n 4-20 --chunks 32 --variants 6 --out gpurun_out/sweep_d.jsonl > gpurun_out/sweep_d.log 2>&1
timeout 900 python scripts/autotune.py --n 28-32 --chunks 32,64,0 --variants 5 --skip-from tuning/sweep_b200_r01c.jsonl --out gpurun_out/sweep_d.jsonl >> gpurun_out/sweep_d.log 2>&1
timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_rtma16 python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline --tune '{"variant":6,"threads_per_block":0,"param":2,"staging":1}' > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_ptmem32 python bench.py --workload c3 --steps 4 --warmup 3 --no-e2e --no-cpu-baseline --tune '{"variant":5,"threads_per_block":128,"param":16,"staging":1}' > /dev/null 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/sweep_d.log
