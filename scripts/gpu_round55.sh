#!/bin/bash
# Round-1 verification of the committed state: GPU suite, smoke, bench C2 (default and short),
# C3, reference arm, ncu launch list of the default bench, ncu capture of RCW n=64 at 1M.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -n 1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_c2_short.json 2> gpurun_out/bench_c2_short.err
timeout 900 python bench.py --workload c3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
python - <<'PY'
import json
for f in ("bench_c2","bench_c2_short","bench_c3","bench_ref"):
    r=json.loads(open("gpurun_out/%s.json"%f).read().strip().splitlines()[-1])
    print(f, r["value"], r.get("roofline",{}) and r["roofline"]["frac"], r.get("clocks"), (r.get("e2e") or {}).get("value"))
PY
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
python scripts/ncu_summary.py launches gpurun_out/launches_c2.csv > gpurun_out/launches_c2.md; head -5 gpurun_out/launches_c2.md
