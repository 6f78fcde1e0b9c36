#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
echo "== default"; timeout 600 python tools/op_micro.py
echo "== HIOS_POOL_OLD"; HIOS_POOL_OLD=1 timeout 600 python tools/op_micro.py i4096_max i4096_avg sq_ nas_avg
echo "== HIOS_DW_OLD"; HIOS_DW_OLD=1 timeout 600 python tools/op_micro.py nas_sep rw_sep
