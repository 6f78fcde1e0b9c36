cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "conv or zoo or end_to_end or bench_config or multi" 2>&1 | tail -3
for v in old new; do
  if [ $v = old ]; then export HIOS_NOPACK=1; else unset HIOS_NOPACK; fi
  echo "== $v"; timeout 300 python tools/op_micro.py sq_conv1 rw_conv1 i4096_conv1a 2>&1 | cut -c1-100
  timeout 900 python bench.py --steps 20 --no-cpu-baseline --sweep "4096,randwire_ws@2048,squeezenet@2048" 2>/dev/null > gpurun_out/b.json; python -c "import json; d=json.loads(open('gpurun_out/b.json').read()); print('bench', round(d['value'],4), {k: (round(v['hios_lp_ms'],3), round(v['cp_frac'],3)) for k,v in d['size_sweep'].items()})"
done
