#!/bin/bash
# ov (overlap-heavy COUNT) sweep on the GPU box: canvas max_dim x probe variant, plus the launch list.
# Usage: bash tools/ov_sweep.sh <tag>   -> gpurun_out/<tag>_*
T=${1:-ovs}
run() { timeout 300 env "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('%.3e pts/s' % d['value'], 'kernel %.3f ms' % d['roofline']['kernel_ms'], d['config'].get('canvas', ''))"; }
for md in 4096 8192 16384 32768; do
  for pipe in -1 0 1; do
    echo -n "max_dim $md pipe $pipe: "; run SPADE_PIPE=$pipe python bench.py --workload ov --max-dim $md --no-e2e --no-cpu-baseline --steps 10 --warmup 3
  done
done > gpurun_out/${T}_sweep.txt 2>&1
echo -n "max_dim 8192 k_agg 0: " >> gpurun_out/${T}_sweep.txt; run SPADE_K_AGG=0 python bench.py --workload ov --no-e2e --no-cpu-baseline --steps 10 --warmup 3 >> gpurun_out/${T}_sweep.txt 2>&1
SPADE_DEBUG_DEFER=1 timeout 300 python bench.py --workload ov --profile --steps 1 --warmup 1 > /dev/null 2> gpurun_out/${T}_defer_stats.txt
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 200 --csv \
    --log-file gpurun_out/${T}_launches_ov.csv python bench.py --workload ov --profile --steps 2 --warmup 1 > /dev/null 2>&1
cat gpurun_out/${T}_sweep.txt
