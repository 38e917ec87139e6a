#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_layout_synth_host.py -q -p no:cacheprovider -k conversion > gpurun_out/pytest_conv.log 2>&1; tail -1 gpurun_out/pytest_conv.log
timeout 900 python scripts/zerocopy_probe.py > gpurun_out/zerocopy.log 2>&1; tail -20 gpurun_out/zerocopy.log
timeout 900 python scripts/c4_sweep.py --no-cusolver --n 1-32 > gpurun_out/c4.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fma.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,smsp__issue_active.avg.pct_of_peak_sustained_active,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum --clock-control none -k regex:potrf --csv --log-file gpurun_out/ncu_winners.csv python scripts/ncu_winners.py --n 1-32 > gpurun_out/ncu_winners.log 2>&1
tail -3 gpurun_out/ncu_winners.log; head -c 300 gpurun_out/ncu_winners.csv
