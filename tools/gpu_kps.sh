echo "== default"; timeout 200 python tools/conv_micro.py --check
echo "== kps1"; HIOS_KPS=1 timeout 200 python tools/conv_micro.py
echo "== kps4"; HIOS_KPS=4 timeout 200 python tools/conv_micro.py --check
