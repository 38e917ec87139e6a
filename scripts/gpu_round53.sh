#!/bin/bash
# bench after factoring the max-over-ranks timing into multi_gpu: plain and torchrun launches.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/b53.json 2> gpurun_out/b53.err; echo "rc=$?"; tail -c 300 gpurun_out/b53.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29521 \
  bench.py --gpus 1 --workload c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b53_c5.json 2> gpurun_out/b53_c5.err; echo "rc=$?"
python - <<'PY'
import json
for f in ("gpurun_out/b53.json","gpurun_out/b53_c5.json"):
    r=json.loads(open(f).read().strip().splitlines()[-1]); print(f, r["value"], r["ms_per_step"], r["roofline"]["frac"], r["clocks"]["samples"])
PY
