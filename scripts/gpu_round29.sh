#!/bin/bash
# RCW (variant 10) first pass: parity, then single-config benches vs QTM/PTMEM.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "rcw or bitwise" > gpurun_out/pytest_rcw.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_rcw.log
tail -n 15 gpurun_out/pytest_rcw.log
for n in 36 40 44 48 52 56 60 64; do
  for k in 1 2; do
    timeout 120 python bench.py --n $n --batch 1048576 --chunk 32 --tune "{\"variant\":10,\"threads_per_block\":256,\"param\":$k,\"staging\":0}" --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import sys,json; r=json.loads(sys.stdin.read()); print($n,$k,r['ms_per_step'],r['hbm_gbs'])" 
  done
done
