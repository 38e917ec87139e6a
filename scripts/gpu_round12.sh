#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_layout_synth_host.py -q -p no:cacheprovider -k host > gpurun_out/pytest_host.log 2>&1; tail -1 gpurun_out/pytest_host.log
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > gpurun_out/clocks_r12.csv 2>&1 &
SMI=$!
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 900 python bench.py --workload c3 --steps 20 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
kill $SMI
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 600 python scripts/solve_bench.py > gpurun_out/solve_bench.log 2>&1
for f in c2 c3 ref; do head -c 300 gpurun_out/bench_$f.json; echo; tail -1 gpurun_out/bench_$f.err; done
tail -12 gpurun_out/solve_bench.log
