#!/bin/bash
# per-op device times (sequential, instrumented graph) for the sizes given
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for spec in "$@"; do
m=${spec%@*}; sz=${spec#*@}
HIOS_DUMP=gpurun_out/ops_${m}_$sz.json timeout 600 python bench.py --model $m --size $sz --steps 10 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/b_${m}_$sz.json 2> gpurun_out/b_${m}_$sz.err; echo rc=$?
python tools/op_table.py gpurun_out/ops_${m}_$sz.json 30
done
