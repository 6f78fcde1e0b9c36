#!/bin/bash
# A/B: committed HEAD build (ab/libhios_head.so) vs the working-tree build:
# op micro-benchmarks ($1: op_micro name prefixes) and the bench (1024 + 4096)
cd "$GRAFT_REPO_ROOT" || exit 1
OPS=${1:-i4096}
for rep in 1 2; do
for v in head cur; do
  if [ $v = head ]; then export HIOS_LIB=$PWD/ab/libhios_head.so; else unset HIOS_LIB; fi
  echo "== $v (rep $rep)"
  timeout 300 python tools/op_micro.py $OPS 2>&1 | cut -c1-90
  timeout 600 python bench.py --steps 20 --no-cpu-baseline --sweep "4096" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench', round(d['value'],4), 'ios', round(d['single_gpu_refs']['ios']['ms'],4), '4096', round(d['size_sweep']['inception_v3@4096']['hios_lp_ms'],3))"
done
done
