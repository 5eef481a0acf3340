#!/bin/bash
# Link an experiment copy of libbqr.so with one translation unit rebuilt
# under extra flags:  tools/mklib_variant.sh <unit.cu> <out.so> <nvcc flags...>
set -e
unit=$1; out=$2; shift 2
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OBJ=$ROOT/paper_conf_ipps_andersonsk12_b200/build_obj
tmp=$(mktemp -d)
(cd $ROOT/paper_conf_ipps_andersonsk12_b200/csrc && nvcc "$@" -O3 -std=c++17 -lineinfo -gencode arch=compute_100a,code=sm_100a \
  -prec-div=true -prec-sqrt=true -ftz=false -fmad=true -Xcompiler -fPIC,-O2 -Xptxas -v -c -o $tmp/u.o $unit 2>&1 | grep -E "spill|Used" | tail -2)
objs=$(ls $OBJ/*.o | grep -v "/${unit%.cu}.o$")
nvcc -shared -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC -o $out $objs $tmp/u.o -lcuda
rm -rf $tmp
