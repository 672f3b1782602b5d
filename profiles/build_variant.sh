#!/bin/bash
# Build an experiment variant of libphoton with extra nvcc defines for k_bbv3.cu (A/B probes, not shipped):
#   profiles/build_variant.sh NAME -DK1_WPC=24 -DK1_NBUF=1   ->  abvar/libphoton_NAME.so
set -e
cd "$(dirname "$0")/.."
name=$1; shift
P=paper_conf_micro_liusc23_b200
FL="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -I include"
mkdir -p abvar/obj_$name
/usr/local/cuda/bin/nvcc $FL "$@" -c $P/csrc/k_bbv3.cu -o abvar/obj_$name/k_bbv3.o
objs=""
for f in $P/_obj/*.o; do b=$(basename $f); if [ "$b" != "k_bbv3.o" ]; then objs="$objs $f"; fi; done
/usr/local/cuda/bin/nvcc -shared -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC $objs abvar/obj_$name/k_bbv3.o \
  -o abvar/libphoton_$name.so -lcudart_static -lrt -ldl -lpthread
echo abvar/libphoton_$name.so
