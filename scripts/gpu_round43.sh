#!/bin/bash
# Copy pipeline with kernel copies over mapped host memory: host tests, bench C2/C3 e2e.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_layout_synth_host.py -q -x -p no:cacheprovider > gpurun_out/pytest_host.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_host.log
tail -n 3 gpurun_out/pytest_host.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 900 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
python - <<'PY'
import json
for f in ("gpurun_out/bench_c2.json","gpurun_out/bench_c3.json"):
    r=json.loads(open(f).read().strip().splitlines()[-1]); e=r["e2e"]
    print(f, r["value"], e["value"], e.get("pcie_gbs_each_way"), {k:(v["value"],v["ms_per_step"]) for k,v in e["paths"].items()})
PY
