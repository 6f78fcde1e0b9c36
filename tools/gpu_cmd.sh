cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "conv or end_to_end or bench_config or multi or tiny" 2>&1 | tail -2
for v in head cur; do
  if [ $v = head ]; then export HIOS_LIB=$PWD/ab/libhios_head.so; else unset HIOS_LIB; fi
  echo "== $v"; timeout 300 python tools/conv_micro.py; timeout 300 python tools/op_micro.py i4096_conv4a i4096_conv2 i4096_6a 2>&1 | cut -c1-60
  timeout 900 python bench.py --steps 30 --no-cpu-baseline --sweep "4096,nasnet_a_large@2048,randwire_ws@2048,squeezenet@2048" 2>/dev/null > gpurun_out/b.json; python -c "import json; d=json.loads(open('gpurun_out/b.json').read()); print('$v bench', round(d['value'],4), 'seq', round(d['single_gpu_refs']['sequential']['ms'],4), 'ios', round(d['single_gpu_refs']['ios']['ms'],4), {k: (round(v['hios_lp_ms'],3), round(v['cp_frac'],3)) for k,v in d['size_sweep'].items()})"
done
