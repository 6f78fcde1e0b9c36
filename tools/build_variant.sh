#!/bin/bash
# build the csrc/ of git revision $1 into ab/libhios_$2.so (A/B timing: HIOS_LIB=ab/libhios_$2.so)
set -e
cd "$(dirname "$0")/.."
rev=$1; name=$2
d=/tmp/hios_variant_$name
rm -rf $d; mkdir -p $d/pkg/csrc $d/build $d/include ab
for f in $(git ls-tree --name-only $rev paper_conf_cluster_kundus23_b200/csrc/); do git show $rev:$f > $d/pkg/csrc/$(basename $f); done
git show $rev:include/hios.h > $d/include/hios.h
HIOS_CSRC=$d/pkg/csrc HIOS_BUILD=$d/build HIOS_LIB_OUT=$PWD/ab/libhios_$name.so python -c "from paper_conf_cluster_kundus23_b200 import build as b; b.build(verbose=True)"
