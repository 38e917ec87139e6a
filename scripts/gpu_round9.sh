#!/bin/bash
# tuned PTMEM table: tests, bench C2/C3/C1/C5, PCIe probe, C4 sweep (new convert), launch list
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -2 gpurun_out/pytest_gpu.log
timeout 120 python scripts/pcie_probe.py > gpurun_out/pcie.json 2>&1; cat gpurun_out/pcie.json
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > gpurun_out/clocks_r9.csv 2>&1 &
SMI=$!
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 900 python bench.py --workload c3 --steps 20 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
timeout 900 python bench.py --workload c1 --steps 50 > gpurun_out/bench_c1.json 2> gpurun_out/bench_c1.err
timeout 1200 python bench.py --workload c5 --steps 3 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
kill $SMI
timeout 1200 python scripts/c4_sweep.py --no-cusolver > gpurun_out/c4.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --workload c3 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
for f in c2 c3 c1 c5; do echo $f; head -c 400 gpurun_out/bench_$f.json; echo; tail -2 gpurun_out/bench_$f.err; done
