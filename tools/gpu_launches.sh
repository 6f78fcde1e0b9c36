#!/bin/bash
# ncu launch lists (cold, serialised) of one timed step per workload
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for m in nasnet_a_large randwire_ws squeezenet; do
HIOS_NCU=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/l_$m.csv python bench.py --model $m --size 2048 --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > gpurun_out/l_$m.out 2>&1; echo ncu_rc=$?
python tools/ncu_summary.py gpurun_out/l_$m.csv
done
