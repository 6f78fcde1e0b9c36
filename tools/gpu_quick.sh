#!/bin/bash
# quick GPU-box check with the in-tree libhios.so (built here, travels with the
# snapshot): GPU tests, step times, per-op table, conv micro-benchmarks.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout -s KILL 900 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.txt
for c in "$@"; do echo "== $c"; timeout -s KILL 900 bash -c "$c"; echo "rc=$?"; done
