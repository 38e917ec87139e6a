#!/bin/bash
# compute-sanitizer on RCW and REGV (memcheck, racecheck, synccheck) via their parity tests.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
SEL="test_rcw_parity_failures_ragged and (41 or 56 or 64) and (32 or 96)"
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "$SEL" > gpurun_out/san_rcw_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/san_rcw_memcheck.log
tail -n 3 gpurun_out/san_rcw_memcheck.log
timeout 1500 compute-sanitizer --tool racecheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "$SEL" > gpurun_out/san_rcw_racecheck.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/san_rcw_racecheck.log
tail -n 3 gpurun_out/san_rcw_racecheck.log
timeout 1500 compute-sanitizer --tool synccheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "$SEL" > gpurun_out/san_rcw_synccheck.log 2>&1; echo "synccheck rc=$?" >> gpurun_out/san_rcw_synccheck.log
tail -n 3 gpurun_out/san_rcw_synccheck.log
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "test_regv_128bit_groups and (4 or 8)" > gpurun_out/san_regv_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/san_regv_memcheck.log
tail -n 3 gpurun_out/san_regv_memcheck.log
