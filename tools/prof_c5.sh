#!/bin/bash
# C5 profiling: launch list (per-kernel device time, DRAM bytes) + ncu --set full of the probe and
# the deferred kernel.  Usage: bash tools/prof_c5.sh <tag> [workload]
T=${1:-p}; W=${2:-c5}
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/${T}_launches_${W}.csv python bench.py --workload $W --profile --steps 2 --warmup 1 > /dev/null 2>&1
echo "launch list rc=$?"
ncu --set full --clock-control none --import-source on -k regex:"k_deferred|k_probe" -s 4 -c 2 \
    -o gpurun_out/${T}_${W}_full python bench.py --workload $W --profile --steps 2 --warmup 1 > gpurun_out/${T}_${W}_ncu.log 2>&1
echo "ncu full rc=$?"; tail -3 gpurun_out/${T}_${W}_ncu.log
