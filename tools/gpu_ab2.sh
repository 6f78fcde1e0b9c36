#!/bin/bash
# full GPU parity + bench A/B ($AB_ENV = the old arm)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -q -x -m gpu > gpurun_out/tg.log 2>&1; echo tg_rc=$?; tail -3 gpurun_out/tg.log
for arm in new old new old; do
  E=""; [ $arm = old ] && E="$AB_ENV"
  env $E timeout 300 python bench.py --no-cpu-baseline --sweep '' --steps 30 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print("bench '$arm'", round(d["value"],4), "seq", round(d["single_gpu_refs"]["sequential"]["ms"],4), "ios", round(d["single_gpu_refs"]["ios_style"]["ms"],4), "conv TF/s", round(d["roofline"]["achieved"],1))'
done
