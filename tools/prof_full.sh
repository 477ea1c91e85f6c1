#!/bin/bash
# ncu --set full of the top probe kernel of each workload (current code); summaries (key metrics,
# stall reasons, top SASS ops by stall) to gpurun_out/<tag>_<w>_ncu.json; reports deleted unless KEEP=1.
#   bash tools/prof_full.sh <tag> "<workloads>"   (c4c = C4's canvas and points with COUNT)
T=$1; WLS=${2:-"c3 c4 c2"}; KREGEX=${KREGEX:-k_probe}
for w in $WLS; do
  args="--workload $w"; [ "$w" = "c4c" ] && args="--workload c4 --count"; [ "$w" = "c2c" ] && args="--workload c2 --count"
  ncu --set full --clock-control none --import-source on -k regex:"$KREGEX" -s 3 -c 1 \
      -o gpurun_out/${T}_${w}_full python bench.py $args --profile --steps 2 --warmup 1 $EXTRA > gpurun_out/${T}_${w}_ncu.log 2>&1
  echo "$w ncu rc=$?"
  python tools/ncu_summary.py gpurun_out/${T}_${w}_full.ncu-rep --json gpurun_out/${T}_${w}_ncu.json --top 20 > /dev/null
  [ -z "$KEEP" ] && rm -f gpurun_out/${T}_${w}_full.ncu-rep
done
