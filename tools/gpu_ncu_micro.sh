#!/bin/bash
# full ncu capture (source-level) of one conv from tools/conv_micro.py: $1 = shape name
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for n in "$@"; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:conv_tc -s 5 -c 1 -o gpurun_out/micro_$n python tools/conv_micro.py $n > gpurun_out/micro_$n.log 2>&1; echo "$n rc=$?"
done
