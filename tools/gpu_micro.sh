echo "== default"; python tools/conv_micro.py --check
echo "== BO=0"; HIOS_BO=0 python tools/conv_micro.py --check 2>&1 | head -4
echo "== nohalo"; HIOS_NOHALO=1 python tools/conv_micro.py
echo "== stages 8"; HIOS_STAGES=8 python tools/conv_micro.py
echo "== ntile 64"; HIOS_NTILE=64 python tools/conv_micro.py
echo "== ntile 128"; HIOS_NTILE=128 python tools/conv_micro.py
