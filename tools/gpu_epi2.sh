#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "conv_parity or end_to_end or zoo or sepconv" > gpurun_out/tq.log 2>&1; echo tq_rc=$?; tail -3 gpurun_out/tq.log
timeout 300 python tools/op_micro.py i4096_conv 2>&1 | cut -c1-90
timeout 900 python bench.py --steps 10 --no-cpu-baseline --sweep "4096,randwire_ws@2048,nasnet_a_large@2048,squeezenet@2048" > gpurun_out/bq.json 2> gpurun_out/bq.err; echo bq_rc=$?
python - <<'PY'
import json
d=json.load(open('gpurun_out/bq.json'))
print('ms', d['value'], 'cp', d['critical_path']['frac'], 'conv', d['roofline']['frac'], 'ios', d['single_gpu_refs'].get('ios'))
for k,v in d['size_sweep'].items():
    print(k, {a: (round(b,3) if isinstance(b,float) else b) for a,b in v.items() if a in ('hios_lp_ms','cp_bound_ms','cp_frac','sequential_ms','error')})
PY
