run() { timeout 300 env "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('%.3e pts/s' % d['value'], 'kernel %.3f ms' % d['roofline']['kernel_ms'])"; }
{ echo -n "multi_agg 0: "; run SPADE_MULTI_AGG=0 python bench.py --workload ov --no-e2e --no-cpu-baseline --steps 10 --warmup 3
  echo -n "count_global 1: "; run SPADE_COUNT_GLOBAL=1 python bench.py --workload ov --no-e2e --no-cpu-baseline --steps 10 --warmup 3
  echo -n "defer 1: "; run SPADE_DEFER=1 python bench.py --workload ov --no-e2e --no-cpu-baseline --steps 10 --warmup 3; } > gpurun_out/ovn_ab.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_probe -s 2 -c 1 -o gpurun_out/ovn_probe \
    python bench.py --workload ov --profile --steps 1 --warmup 2 > gpurun_out/ovn_ncu.log 2>&1
cat gpurun_out/ovn_ab.txt
