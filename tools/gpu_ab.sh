#!/bin/bash
# same-box A/B of the in-tree libhios.so against ab/libhios_$1.so (tools/build_variant.sh)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
B=ab/libhios_$1.so
for rep in 1 2; do
  for lib in in-tree $B; do
    if [ $lib = in-tree ]; then unset HIOS_LIB; else export HIOS_LIB=$PWD/$lib; fi
    timeout 300 python tools/step_time.py --size 1024 --windows 1,5 2>&1 | grep -v Warn
    timeout 300 python tools/step_time.py --size 4096 --windows 5 2>&1 | grep -v Warn
  done
done
unset HIOS_LIB
S="tiny1x1 7c_pool 6a_s2 4a 3b_4096 5b1x1_4096 2a_4096 2b_4096 4a_4096 7c1x1_4096"
echo "A (in-tree)"; timeout 300 python tools/conv_micro.py $S 2>&1 | grep -v Warn
echo "B ($B)"; HIOS_LIB=$PWD/$B timeout 300 python tools/conv_micro.py $S 2>&1 | grep -v Warn
