#!/bin/bash
# Build a libspade.so variant with extra nvcc flags for probe.cu (A/B runs; the other objects are the
# in-tree build's: run the in-tree build first).  Usage: tools/build_variant.sh out.so "-DSPADE_PROBE_T=768 ..."
set -e
R=$(cd "$(dirname "$0")/.." && pwd); C=$R/paper_conf_icde_doraiswamyf22_b200/csrc
OUT=$1; FLAGS=$2; T=$(mktemp -d)
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr -Xcompiler -fPIC,-fvisibility=hidden"
nvcc $F $FLAGS -I $R/include -dc -o $T/probe.o $C/probe.cu > $T/log 2>&1 || { cat $T/log; exit 1; }
nvcc -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC -dlink -o $T/probe_dlink.o $T/probe.o
g++ -shared -fPIC -o $OUT $C/spade_api.o $C/canvas_build.o $T/probe.o $T/probe_dlink.o $C/knn.o $C/polygon_join.o $C/layers.o \
    -L/usr/local/cuda/lib64 -lcudadevrt -lcudart_static -lrt -lpthread -ldl
rm -rf $T
