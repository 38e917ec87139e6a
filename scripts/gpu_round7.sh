#!/bin/bash
# smem opt-in fix: bitwise parity, sweep RTMA (all n) + PTMEM S=24, bench C2/C3 (zero-copy e2e), C4 sweep
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python scripts/autotune.py --n 4-20 --chunks 32 --variants 6 --out gpurun_out/sweep_e.jsonl > gpurun_out/sweep_e.log 2>&1
timeout 900 python scripts/autotune.py --n 28-32 --chunks 32,64,0 --variants 5 --skip-from tuning/sweep_b200_r01c.jsonl --out gpurun_out/sweep_e.jsonl >> gpurun_out/sweep_e.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 900 python bench.py --workload c3 --steps 20 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
timeout 1200 python scripts/c4_sweep.py > gpurun_out/c4.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_ptmem32 python bench.py --workload c3 --steps 4 --warmup 3 --no-e2e --no-cpu-baseline --tune '{"variant":5,"threads_per_block":128,"param":16,"staging":1}' > gpurun_out/prof_ptmem32.out 2>&1
tail -2 gpurun_out/sweep_e.log; cat gpurun_out/bench_c2.json; cat gpurun_out/bench_c3.json; tail -3 gpurun_out/c4.log
