#!/bin/bash
# One profiling pass for profiles/: the default bench line (C3), bench lines of the other
# workloads, the ncu launch list of the C3 bench command, one ncu --set full of C3's k_probe and
# of C5's probe + deferred kernels.
# Usage (on the GPU box): bash tools/profile_round.sh <tag>    -> gpurun_out/<tag>_*
T=${1:-prof}
python bench.py > gpurun_out/${T}_bench_c3.json 2> gpurun_out/${T}_bench_c3.err
for wl in c2 c4 c5 dj dj2 knn ov; do
  python bench.py --workload $wl --no-e2e --steps 20 --warmup 3 --cpu-seconds 8 > gpurun_out/${T}_bench_$wl.json 2> gpurun_out/${T}_bench_$wl.err
done
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${T}_launches_c3.csv \
    python bench.py --profile --steps 5 --warmup 3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_probe -s 3 -c 1 -o gpurun_out/${T}_probe_c3 \
    python bench.py --profile --steps 1 --warmup 3 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:"k_probe|k_deferred|k_fixup|k_move" -c 12 --csv --log-file gpurun_out/${T}_launches_c5_c4.csv \
    bash -c "python bench.py --workload c5 --profile --steps 2 --warmup 1; python bench.py --workload c4 --profile --steps 2 --warmup 1" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_probe|k_deferred" -s 2 -c 2 -o gpurun_out/${T}_c5 \
    python bench.py --workload c5 --profile --steps 1 --warmup 1 > /dev/null 2>&1
ls -la gpurun_out
