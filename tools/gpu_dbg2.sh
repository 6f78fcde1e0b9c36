#!/bin/bash
# conv bottleneck experiments: HIOS_DBG bits 2 = no B/stage loads, 4 = no halo A loads,
# 8 = no MMAs, 16 = no epilogue work (results are garbage; timing only)
cd "$GRAFT_REPO_ROOT" || exit 1
for d in 0 2 4 6 8 16 22 24 12; do
echo "== HIOS_DBG=$d"; HIOS_DBG=$d timeout 300 python tools/op_micro.py i4096_conv 2>&1 | cut -c1-60
done
echo "== pools"; timeout 300 python tools/op_micro.py i4096_max i4096_avg sq_ nas_avg nas_sep rw_sep
