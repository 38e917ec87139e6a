#!/bin/bash
# synccheck triage: does it flag every tcgen05.alloc kernel (PTMEM cp.async path, QTM) or only RCW?
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 compute-sanitizer --tool synccheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "test_qtm_parity_failures_ragged and 33 and 32" > gpurun_out/san_qtm_sync.log 2>&1
grep -E "ERROR SUMMARY|Barrier error|at void" gpurun_out/san_qtm_sync.log | sort | uniq -c | head
timeout 900 compute-sanitizer --tool synccheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "test_parity_chunk32_ragged and 24" > gpurun_out/san_ptmem_sync.log 2>&1
grep -E "ERROR SUMMARY|Barrier error|at void" gpurun_out/san_ptmem_sync.log | sort | uniq -c | head
timeout 900 compute-sanitizer --tool synccheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "test_rcw_parity_failures_ragged and 64 and 32" > gpurun_out/san_rcw64_sync.log 2>&1
grep -E "ERROR SUMMARY|Barrier error|at void" gpurun_out/san_rcw64_sync.log | sort | uniq -c | head
