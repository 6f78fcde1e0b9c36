echo "== default"; timeout 120 python tools/conv_micro.py
for nt in 64 128 256; do for nm in 1 4; do echo "== NTILE $nt NMMA $nm"; HIOS_NMMA=$nm HIOS_NTILE=$nt timeout 120 python tools/conv_micro.py; done; done
