#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
for d in 0 16 32 64 96; do echo "== HIOS_DBG=$d"; HIOS_DBG=$d timeout 300 python tools/op_micro.py i4096_conv3b i4096_conv2b 2>&1 | cut -c1-70; done
echo "== no TMA store"; HIOS_NOTMASTORE=1 timeout 300 python tools/op_micro.py i4096_conv3b i4096_conv2b 2>&1 | cut -c1-70
