cd $GRAFT_REPO_ROOT
for o in 1 2; do echo "== OCC $o"; HIOS_OCC=$o timeout 300 python tools/op_micro.py i4096_conv 2>&1 | cut -c1-90; HIOS_OCC=$o timeout 300 python tools/conv_micro.py; done
