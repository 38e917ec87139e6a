#!/bin/bash
# Round-2 job 34: branch-free sqrt/rcp in REG / RTMA / PANEL -- full GPU suite
# and the per-n block n = 1..32 (short bench).
cd "$GRAFT_REPO_ROOT" || exit 1
TAG=${1:-j34}; shift
O=gpurun_out/$TAG; mkdir -p $O
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -n 4 $O/pytest_gpu.log
timeout 900 python bench.py --workload c2 --steps 5 --warmup 3 --per-n 1-32 --no-e2e --no-cpu-baseline > $O/bench_pern.json 2> $O/bench_pern.err; echo "pern rc=$?"
python scripts/per_n_table.py $O/bench_pern.json > $O/per_n.md
