cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "pool or zoo or end_to_end" 2>&1 | tail -2
for v in head cur; do
  if [ $v = head ]; then export HIOS_LIB=$PWD/ab/libhios_head.so; else unset HIOS_LIB; fi
  echo "== $v"; timeout 300 python tools/op_micro.py i4096_avgpool nas_avg 2>&1 | cut -c1-100
  timeout 900 python bench.py --steps 30 --no-cpu-baseline --sweep "4096,nasnet_a_large@2048" 2>/dev/null > gpurun_out/b.json; python -c "import json; d=json.loads(open('gpurun_out/b.json').read()); print('$v bench', round(d['value'],4), {k: (round(v['hios_lp_ms'],3), round(v['cp_frac'],3)) for k,v in d['size_sweep'].items()})"
done
