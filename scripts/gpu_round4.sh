#!/bin/bash
# tuned table: bench C2/C3, ncu of both bench kernels, launch list
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/clocks_r4.csv 2>&1 &
SMI=$!
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 900 python bench.py --workload c3 --steps 20 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
kill $SMI
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_c2_r4 python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_c2.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_c3_r4 python bench.py --workload c3 --steps 4 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_c3.out 2>&1
cat gpurun_out/bench_c2.json gpurun_out/bench_c3.json; tail -2 gpurun_out/bench_c2.err gpurun_out/bench_c3.err
