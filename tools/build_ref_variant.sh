#!/bin/bash
# build_variants/<name>.so from the csrc/ of git revision <rev> (A/B baselines)
# usage: tools/build_ref_variant.sh <rev> <name> [extra nvcc flags]
set -e
REV=$1; NAME=$2; shift 2
ROOT=$(cd $(dirname $0)/.. && pwd)
T0=$(mktemp -d)
mkdir -p $T0/pkg/csrc $T0/include $ROOT/build_variants        # csrc/../../include as in the tree
for f in $(git -C $ROOT ls-tree --name-only $REV paper_conf_sc_huangd0lc23_b200/csrc/); do git -C $ROOT show $REV:$f > $T0/pkg/csrc/$(basename $f); done
git -C $ROOT show $REV:include/cuszp.h > $T0/include/cuszp.h
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -fmad=false -prec-div=true -prec-sqrt=true -ftz=false -Xcompiler -fPIC -Xcompiler -O2 --cudart static -I $T0/include "$@" -shared -o $ROOT/build_variants/$NAME.so $T0/pkg/csrc/*.cu
rm -rf $T0
echo $ROOT/build_variants/$NAME.so
