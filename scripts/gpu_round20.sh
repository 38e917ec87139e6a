#!/bin/bash
# New warp-tile conversion kernel: parity + C4 conversion bandwidth; zero-copy probe at n=16.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_layout_synth_host.py -q -x -p no:cacheprovider > gpurun_out/pytest_conv.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_conv.log
tail -n 3 gpurun_out/pytest_conv.log
timeout 900 python scripts/c4_sweep.py --no-cusolver --n 1-64 --out gpurun_out/c4_conv.jsonl --md gpurun_out/c4_conv.md > gpurun_out/c4.log 2>&1
python - <<'PY'
import json
for l in open('gpurun_out/c4_conv.jsonl'):
    r=json.loads(l); print(r['n'], round(r['convert_gbs']), end='; ')
print()
PY
timeout 600 python scripts/zerocopy_probe.py > gpurun_out/zc.log 2>&1; tail -n 12 gpurun_out/zc.log
