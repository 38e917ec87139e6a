#!/bin/bash
# Round-2 job 31: branch-free sqrt/rcp in every kernel -- exhaustive bitwise
# check against the intrinsics, full GPU suite, default bench (C3 + per-n).
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j31}; shift
O=gpurun_out/$TAG; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include scripts/r02/verify_fast_sqrt_rcp.cu -o /tmp/vfsr && timeout 300 /tmp/vfsr > $O/verify.json; echo "verify rc=$?"; cat $O/verify.json
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -n 3 $O/pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
