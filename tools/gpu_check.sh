#!/bin/bash
# full GPU test suite + default bench line (state check)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 1200 python -m pytest tests -q -x -m gpu > gpurun_out/tgpu.log 2>&1; echo tgpu_rc=$?; tail -5 gpurun_out/tgpu.log
timeout 600 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -3 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo bench_rc=$?
tail -c 1500 gpurun_out/bench_full.json; tail -5 gpurun_out/bench_full.err
