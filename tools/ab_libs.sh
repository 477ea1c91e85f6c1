#!/bin/bash
# A/B different builds of libspade.so: tools/ab_libs.sh lib1.so lib2.so ...  (restores the original)
cp paper_conf_icde_doraiswamyf22_b200/libspade.so /tmp/libspade_orig.so
for L in "$@"; do
  cp "$L" paper_conf_icde_doraiswamyf22_b200/libspade.so
  echo "== $L"; VARIANTS=${VARIANTS:-0} ./tools/tune_probe.sh $BENCH_ARGS
done
cp /tmp/libspade_orig.so paper_conf_icde_doraiswamyf22_b200/libspade.so
