#!/bin/bash
# Final pass: GPU suite, smoke, every bench workload (short), reference arm.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -n 1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
for wl in c1 c2i c3 c4n48 c4n64; do
  timeout 900 python bench.py --workload $wl --steps 10 --warmup 3 --cpu-seconds 4 > gpurun_out/bench_$wl.json 2> gpurun_out/bench_$wl.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
python - <<'PY'
import json
for f in ("c2","c1","c2i","c3","c4n48","c4n64","ref"):
    try:
        r=json.loads(open("gpurun_out/bench_%s.json"%f).read().strip().splitlines()[-1])
        print(f, r["value"], r["unit"], (r.get("roofline") or {}).get("frac"), (r.get("e2e") or {}).get("value"), (r.get("cpu_baseline") or {}).get("value"), r.get("clocks",{}) and r["clocks"].get("sm_mhz"))
    except Exception as e:
        print(f, "ERR", e)
PY
