#!/bin/bash
# per-op device times (sequential, instrumented graph) at 2048^2 and 4096^2
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for sz in 4096 2048; do
HIOS_DUMP=gpurun_out/ops_$sz.json timeout 600 python bench.py --size $sz --steps 10 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/b_$sz.json 2> gpurun_out/b_$sz.err; echo rc=$?
tail -c 800 gpurun_out/b_$sz.json; tail -3 gpurun_out/b_$sz.err
done
for m in randwire_ws nasnet_a_large squeezenet; do
HIOS_DUMP=gpurun_out/ops_${m}.json timeout 900 python bench.py --model $m --size 2048 --steps 10 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/b_$m.json 2> gpurun_out/b_$m.err; echo rc=$?
tail -c 600 gpurun_out/b_$m.json; tail -3 gpurun_out/b_$m.err
done
