cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "pool or zoo or end_to_end" 2>&1 | tail -2
timeout 900 python bench.py --steps 30 --no-cpu-baseline 2>/dev/null > gpurun_out/b.json; python -c "import json; d=json.loads(open('gpurun_out/b.json').read()); print('bench', round(d['value'],4), {k: (round(v['hios_lp_ms'],3), round(v['cp_frac'],3)) for k,v in d['size_sweep'].items()})"
