echo "== occ1"; timeout 120 python tools/conv_micro.py
echo "== occ2"; HIOS_OCC=2 timeout 120 python tools/conv_micro.py --check
echo "== occ2 nt64"; HIOS_OCC=2 HIOS_NTILE=64 timeout 120 python tools/conv_micro.py
echo "== occ2 nt128"; HIOS_OCC=2 HIOS_NTILE=128 timeout 120 python tools/conv_micro.py
