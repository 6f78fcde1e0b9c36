#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
for cfg in "148 6" "74 8" "148 8" "96 8" "48 8" "148 6"; do
  set -- $cfg
  HIOS_SPLIT_CTAS=$1 HIOS_SPLIT_MINK=$2 timeout 300 python bench.py --no-cpu-baseline --sweep "" --steps 30 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(\"ctas $1 mink $2 bench\", round(d[\"value\"],4), \"seq\", round(d[\"single_gpu_refs\"][\"sequential\"][\"ms\"],4))"
done
HIOS_NOSPLIT=1 timeout 300 python bench.py --no-cpu-baseline --sweep "" --steps 30 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(\"nosplit bench\", round(d[\"value\"],4), \"seq\", round(d[\"single_gpu_refs\"][\"sequential\"][\"ms\"],4))"
