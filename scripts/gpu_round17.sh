#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 10 python -m pytest tests/test_gpu_solve.py tests/test_gpu_layout_synth_host.py -q -p no:cacheprovider -k "conversion or (sposv and 16) or host_end_to_end" > gpurun_out/sanitizer_memcheck3.log 2>&1; echo "memcheck3 rc=$?" >> gpurun_out/sanitizer_memcheck3.log
tail -3 gpurun_out/sanitizer_memcheck3.log
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 10 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "bitwise_identical and (32- or 40- or 44- or 36-)" > gpurun_out/sanitizer_memcheck4.log 2>&1; echo "memcheck4 rc=$?" >> gpurun_out/sanitizer_memcheck4.log
tail -3 gpurun_out/sanitizer_memcheck4.log
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -2 gpurun_out/pytest_gpu.log
timeout 1800 python scripts/c4_sweep.py > gpurun_out/c4.log 2>&1
tail -3 gpurun_out/c4.log
