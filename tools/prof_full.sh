#!/bin/bash
# ncu --set full of the top probe kernel of each workload (current code):
#   bash tools/prof_full.sh <tag> "<workloads>"   (c4c = C4's canvas and points with COUNT)
T=$1; WLS=${2:-"c3 c4 c2"}
for w in $WLS; do
  args="--workload $w"; [ "$w" = "c4c" ] && args="--workload c4 --count"
  ncu --set full --clock-control none --import-source on -k regex:"k_probe" -s 3 -c 1 \
      -o gpurun_out/${T}_${w}_full python bench.py $args --profile --steps 2 --warmup 1 > gpurun_out/${T}_${w}_ncu.log 2>&1
  echo "$w ncu rc=$?"
done
