#!/bin/bash
# A/B of prebuilt library variants: bash tools/ab_libs3.sh <tag> "<workloads>" lib1.so lib2.so ...
T=$1; WLS=$2; shift 2
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
cp paper_conf_icde_doraiswamyf22_b200/libspade.so /tmp/libspade_orig.so
for L in /tmp/libspade_orig.so "$@"; do
  cp "$L" paper_conf_icde_doraiswamyf22_b200/libspade.so
  for w in $WLS; do
    timeout 600 python bench.py --workload $w --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --no-parity 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$(basename $L)', '$w', f\"{d['ms_per_step']:.3f} ms frac {d['roofline']['frac']:.3f}\", d['check'])" || echo "$L $w FAILED"
  done
done | tee gpurun_out/${T}_abl.txt
cp /tmp/libspade_orig.so paper_conf_icde_doraiswamyf22_b200/libspade.so
