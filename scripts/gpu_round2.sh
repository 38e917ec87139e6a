#!/bin/bash
# autotune sweep + ncu captures of the bench kernels
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python - > gpurun_out/nvml_latency.txt 2>&1 <<'PY'
import time, pynvml
pynvml.nvmlInit(); h=pynvml.nvmlDeviceGetHandleByIndex(0)
for name in ("nvmlDeviceGetClockInfo","nvmlDeviceGetCurrentClocksEventReasons","nvmlDeviceGetCurrentClocksThrottleReasons"):
    fn=getattr(pynvml,name,None)
    if fn is None: print(name,"missing"); continue
    t=time.perf_counter(); 
    for _ in range(100): fn(h, pynvml.NVML_CLOCK_SM) if name=="nvmlDeviceGetClockInfo" else fn(h)
    print(name, (time.perf_counter()-t)/100*1e3, "ms")
PY
timeout 1200 python scripts/autotune.py --n 1-32 --chunks 32,64,128,256,512,0 --out gpurun_out/sweep.jsonl > gpurun_out/sweep.log 2>&1
timeout 900 python scripts/autotune.py --n 33-64 --chunks 32,0 --out gpurun_out/sweep.jsonl >> gpurun_out/sweep.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/launches_c2.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_c2 python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_c2.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf -s 3 -c 1 -o gpurun_out/prof_c3 python bench.py --workload c3 --steps 4 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_c3.out 2>&1
timeout 600 python bench.py --workload c3 --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
tail -3 gpurun_out/sweep.log; cat gpurun_out/nvml_latency.txt; cat gpurun_out/bench_c3.json; tail -2 gpurun_out/bench_c3.err; ls -la gpurun_out
