#!/bin/bash
# The launch path the driver uses for N>1 (torchrun, NCCL), here with one rank: C2 and C5.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 \
  bench.py --gpus 1 --steps 10 --warmup 3 > gpurun_out/trun_c2.json 2> gpurun_out/trun_c2.err; echo "rc=$?"; tail -c 700 gpurun_out/trun_c2.json
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29512 \
  bench.py --gpus 1 --workload c5 --steps 5 --warmup 3 --no-e2e > gpurun_out/trun_c5.json 2> gpurun_out/trun_c5.err; echo "rc=$?"; tail -c 900 gpurun_out/trun_c5.json
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29513 \
  bench.py --impl reference --gpus 1 --steps 3 --warmup 3 > gpurun_out/trun_ref.json 2> gpurun_out/trun_ref.err; echo "rc=$?"; tail -c 300 gpurun_out/trun_ref.json
