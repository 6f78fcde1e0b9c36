cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
for v in old new; do
  if [ $v = old ]; then export HIOS_NOCHANPAD=1; else unset HIOS_NOCHANPAD; fi
  echo "== $v"; timeout 300 python tools/op_micro.py i4096_conv rw_conv nas_sep rw_sep 2>&1 | cut -c1-100; timeout 300 python tools/conv_micro.py
  timeout 900 python bench.py --steps 20 --no-cpu-baseline 2>/dev/null > gpurun_out/b.json; python -c "import json; d=json.loads(open('gpurun_out/b.json').read()); print('bench', round(d['value'],4), {k: (round(v['hios_lp_ms'],3), round(v['cp_frac'],3)) for k,v in d['size_sweep'].items()})"
done
