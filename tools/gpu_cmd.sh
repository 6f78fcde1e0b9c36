cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "conv or inception or tiny or squeeze" 2>&1 | tail -3
timeout 600 python tools/conv_trace2.py i4096_conv1a i4096_conv3b 2>&1 | tail -40
for e in 2 1; do echo "== EPI $e"; HIOS_EPI=$e timeout 300 python tools/op_micro.py i4096_conv 2>&1 | cut -c1-90; done
HIOS_LIB=$PWD/ab/libhios_head.so timeout 600 python bench.py --steps 20 --no-cpu-baseline --sweep "4096" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('HEAD bench', round(d['value'],4), 'ios', round(d['single_gpu_refs']['ios']['ms'],4), '4096', round(d['size_sweep']['inception_v3@4096']['hios_lp_ms'],3))"
for e in 2 1; do
HIOS_EPI=$e timeout 600 python bench.py --steps 20 --no-cpu-baseline --sweep "4096" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('EPI$e bench', round(d['value'],4), 'ios', round(d['single_gpu_refs']['ios']['ms'],4), '4096', round(d['size_sweep']['inception_v3@4096']['hios_lp_ms'],3))"
done
timeout 600 python bench.py --steps 20 --no-cpu-baseline --sweep "4096" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('default bench', round(d['value'],4), 'ios', round(d['single_gpu_refs']['ios']['ms'],4), '4096', round(d['size_sweep']['inception_v3@4096']['hios_lp_ms'],3))"
