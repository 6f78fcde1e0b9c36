echo "== default"; timeout 200 python tools/conv_micro.py
echo "== occ2"; HIOS_OCC=2 timeout 200 python tools/conv_micro.py
echo "== occ2 nt64"; HIOS_OCC=2 HIOS_NTILE=64 timeout 200 python tools/conv_micro.py
echo "== nt256"; HIOS_NTILE=256 timeout 200 python tools/conv_micro.py
echo "== nt128 nmma1"; HIOS_NTILE=128 HIOS_NMMA=1 timeout 200 python tools/conv_micro.py
