#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python tools/fig1_contention.py --out gpurun_out/fig1.json 2>&1 | tail -25
timeout 300 python tools/conv_trace.py 7c_1x1 6e_1x7 7c_3x3 6e_1x1 2>&1 | tail -60
