#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "conv_parity or pool or sepconv or zoo" > gpurun_out/tq.log 2>&1; echo tq_rc=$?; tail -3 gpurun_out/tq.log
echo "== default"; timeout 600 python tools/op_micro.py
echo "== HIOS_POOL_OLD"; HIOS_POOL_OLD=1 timeout 600 python tools/op_micro.py i4096_max i4096_avg sq_ nas_avg
