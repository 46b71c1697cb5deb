#!/bin/bash
# build a tuning variant of libefg.so: tools/build_variant.sh NAME "-DEFG_STAGE_BYTES=8192 ..."
set -e
NAME=$1; DEFS=$2
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OUT=$ROOT/build/var_$NAME; mkdir -p $OUT
CS=$ROOT/paper_conf_ipps_gerak23_b200/csrc
F="-gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I $ROOT/include -I $CS -Xcompiler -fPIC,-fopenmp -lineinfo $DEFS"
for s in $(cd $CS && ls *.cu *.cpp); do
  nvcc $F -c $CS/$s -o $OUT/$s.o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $OUT/libefg.so $OUT/*.o -Xcompiler -fopenmp -lgomp
echo $OUT/libefg.so
