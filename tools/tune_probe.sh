#!/bin/bash
# Probe launch-shape sweep on the GPU box: one bench line per SPADE_PROBE_VARIANT.
for v in ${VARIANTS:-0 1 2 3 4}; do
  SPADE_PROBE_VARIANT=$v python bench.py --no-e2e --no-cpu-baseline --steps ${STEPS:-40} --warmup 5 "$@" 2>/dev/null \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('variant', $v, '%.3e pts/s' % d['value'], 'kernel %.3f ms' % d['roofline']['kernel_ms'], 'frac %.3f' % d['roofline']['frac'], d['check'])"
done
