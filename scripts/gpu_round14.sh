#!/bin/bash
# compute-sanitizer memcheck / racecheck on the parity suite (small sizes)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
SEL="test_parity_chunk32_ragged and (4 or 16 or 20 or 24 or 29 or 32 or 40)"
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "$SEL" > gpurun_out/sanitizer_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/sanitizer_memcheck.log
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "bitwise_identical and (16-32 or 32-32 or 24-32 or 20-0)" > gpurun_out/sanitizer_memcheck2.log 2>&1; echo "memcheck2 rc=$?" >> gpurun_out/sanitizer_memcheck2.log
timeout 1500 compute-sanitizer --tool racecheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "test_parity_chunk32_ragged and (20 or 24 or 32)" > gpurun_out/sanitizer_racecheck.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/sanitizer_racecheck.log
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_solve.py tests/test_gpu_layout_synth_host.py -q -p no:cacheprovider -k "conversion or (sposv and 16) or host_end_to_end" > gpurun_out/sanitizer_memcheck3.log 2>&1; echo "memcheck3 rc=$?" >> gpurun_out/sanitizer_memcheck3.log
for f in gpurun_out/sanitizer_*.log; do echo == $f; tail -4 $f; done
