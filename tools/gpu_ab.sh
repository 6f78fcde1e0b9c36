#!/bin/bash
# A/B of a conv-kernel change: parity subset, micro (both arms), trace, bench (both arms)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "conv_parity or tiny or zoo or end_to_end_bf16" > gpurun_out/tq.log 2>&1; echo tq_rc=$?; tail -3 gpurun_out/tq.log
echo "== micro new"; timeout 300 python tools/conv_micro.py --check
echo "== micro old ($AB_ENV)"; env $AB_ENV timeout 300 python tools/conv_micro.py
timeout 300 python tools/conv_trace.py 6e_1x1 7c_3x3 2>&1 | grep -E "==|epi:|start|tma0|data0|mma_end|exit"
for arm in new old; do
  E=""; [ $arm = old ] && E="$AB_ENV"
  env $E timeout 300 python bench.py --no-cpu-baseline --sweep '' --steps 30 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print("bench '$arm'", round(d["value"],4), "seq", round(d["single_gpu_refs"]["sequential"]["ms"],4), "conv TF/s", round(d["roofline"]["achieved"],1))'
done
