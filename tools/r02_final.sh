#!/bin/bash
# End-of-round measurement of the committed code (one B200): GPU tests, smoke, every workload's
# bench line, the ncu launch list of the default bench command, ncu --set full summaries of the
# C3 / C5 probe kernels and DRAM bytes per launch of C3 / C4 / C5.  Usage: bash tools/r02_final.sh <tag>
T=${1:-fin}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${T}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/${T}_smoke.log
bash tools/r02_matrix.sh ${T}
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${T}_launches_c3.csv \
    python bench.py --profile --steps 5 --warmup 3 > /dev/null 2>&1; echo "launch list rc=$?"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none \
    -k regex:"k_probe|k_deferred|k_fixup|k_move|k_multi" -c 30 --csv --log-file gpurun_out/${T}_launches_dram.csv \
    bash -c "python bench.py --workload c3 --profile --steps 2 --warmup 1; python bench.py --workload c4 --profile --steps 2 --warmup 1; python bench.py --workload c5 --profile --steps 2 --warmup 1; python bench.py --workload c2 --profile --steps 2 --warmup 1" > /dev/null 2>&1; echo "dram list rc=$?"
for w in c3 c5; do
  ncu --set full --clock-control none --import-source on -k regex:"k_probe" -s 3 -c 1 -o gpurun_out/${T}_${w}_full \
      python bench.py --workload $w --profile --steps 2 --warmup 1 > /dev/null 2>&1; echo "$w ncu rc=$?"
  python tools/ncu_summary.py gpurun_out/${T}_${w}_full.ncu-rep --json gpurun_out/${T}_${w}_ncu.json --top 20 > /dev/null 2>&1
  python tools/ncu_lines.py gpurun_out/${T}_${w}_full.ncu-rep > gpurun_out/${T}_${w}_lines.txt 2>/dev/null
  rm -f gpurun_out/${T}_${w}_full.ncu-rep
done
ls gpurun_out | grep "^${T}_"
