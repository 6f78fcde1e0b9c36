#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
./tools/mma_bench3 > gpurun_out/mma3.txt 2>&1; cat gpurun_out/mma3.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "pool or sepconv" > gpurun_out/tq.log 2>&1; echo tq_rc=$?; tail -3 gpurun_out/tq.log
for v in 0 1; do
if [ $v = 1 ]; then export HIOS_POOL_OLD=1; fi
timeout 900 python bench.py --steps 10 --no-cpu-baseline --sweep "4096,nasnet_a_large@2048,squeezenet@2048" > gpurun_out/bq$v.json 2> gpurun_out/bq$v.err; echo bq_rc=$?
python - $v <<'PY'
import json,sys
d=json.load(open(f'gpurun_out/bq{sys.argv[1]}.json'))
print('POOL_OLD' if sys.argv[1]=='1' else 'tiled', 'ms', d['value'], 'cp', d['critical_path']['frac'])
for k,v in d['size_sweep'].items():
    print(k, {a: (round(b,3) if isinstance(b,float) else b) for a,b in v.items() if a in ('hios_lp_ms','cp_bound_ms','cp_frac','sequential_ms','error')})
PY
done
