#!/bin/bash
# A/B builds of libspade.so over workloads: WLS="c5 dj2" bash tools/ab_libs2.sh a.so b.so ...
cp paper_conf_icde_doraiswamyf22_b200/libspade.so /tmp/libspade_orig.so
for L in "$@"; do
  cp "$L" paper_conf_icde_doraiswamyf22_b200/libspade.so
  echo "== $L"; WLS="${WLS:-c5}" STEPS=${STEPS:-10} bash tools/bench_matrix.sh
done
cp /tmp/libspade_orig.so paper_conf_icde_doraiswamyf22_b200/libspade.so
