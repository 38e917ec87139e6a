#!/bin/bash
# Table with RCW: full GPU suite, smoke, C4 n-sweep, bench C2/C3, and a bench at n=64.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -n 2 gpurun_out/smoke.log
timeout 1800 python scripts/c4_sweep.py --out gpurun_out/c4_r39.jsonl --md gpurun_out/c4_r39.md > gpurun_out/c4.log 2>&1
tail -n 2 gpurun_out/c4.log
timeout 600 python bench.py --n 64 --batch 1048576 --chunk 32 --no-cpu-baseline > gpurun_out/bench_n64.json 2> gpurun_out/bench_n64.err; tail -c 400 gpurun_out/bench_n64.json
