echo "== default"; timeout 200 python tools/conv_micro.py --check
echo "== cap128"; HIOS_TAPCAP=128 timeout 200 python tools/conv_micro.py
echo "== nosplit"; HIOS_NOSPLIT=1 timeout 200 python tools/conv_micro.py
for w in 4; do timeout 300 python bench.py --no-cpu-baseline --sweep '' --steps 20 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print("bench", round(d["value"],4), d["single_gpu_refs"]["sequential"]["ms"])'; done
HIOS_TAPCAP=128 timeout 300 python bench.py --no-cpu-baseline --sweep '' --steps 20 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print("bench cap128", round(d["value"],4), d["single_gpu_refs"]["sequential"]["ms"])'
