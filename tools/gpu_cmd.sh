cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "conv or end_to_end or bench_config" 2>&1 | tail -2
for d in 32 0; do echo "== DBG $d"; HIOS_DBG=$d timeout 300 python tools/op_micro.py i4096_conv sq_conv1 rw_conv1 2>&1 | cut -c1-60; HIOS_DBG=$d timeout 300 python tools/conv_trace2.py i4096_conv2a 2>&1 | sed -n 2,6p; done
timeout 900 python bench.py --steps 20 --no-cpu-baseline 2>/dev/null > gpurun_out/b.json; python -c "import json; d=json.loads(open('gpurun_out/b.json').read()); print('bench', round(d['value'],4), {k: (round(v['hios_lp_ms'],3), round(v['cp_frac'],3)) for k,v in d['size_sweep'].items()})"
