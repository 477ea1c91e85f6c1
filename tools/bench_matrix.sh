#!/bin/bash
# Run bench.py over workloads (WLS) and print one summary line each; extra args go to bench.py.
for wl in ${WLS:-c3}; do
  python bench.py --workload $wl --no-e2e --no-cpu-baseline --steps ${STEPS:-20} --warmup 3 "$@" > /tmp/bm_$wl.json 2>/tmp/bm_$wl.err \
  && python -c "import json; d=json.load(open('/tmp/bm_$wl.json')); r=d['roofline']; print('$wl', '%.3e pts/s' % d['value'], 'kernel %.3f ms' % r['kernel_ms'], 'frac %.3f' % r['frac'], d['check'])" \
  || tail -3 /tmp/bm_$wl.err
done
