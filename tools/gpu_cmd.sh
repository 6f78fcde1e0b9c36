cd $GRAFT_REPO_ROOT
for w in 5 6 8 4 5; do
  timeout 900 python bench.py --steps 30 --window $w --no-cpu-baseline --sweep "4096" 2>/dev/null > gpurun_out/b.json; python -c "import json; d=json.loads(open('gpurun_out/b.json').read()); print('w=$w bench', round(d['value'],4), 'pred', d['schedule']['predicted_ms'], 'ios', round(d['single_gpu_refs']['ios']['ms'],4), {k: (round(v['hios_lp_ms'],3), round(v['cp_frac'],3)) for k,v in d['size_sweep'].items()})"
done
