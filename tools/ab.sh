#!/bin/bash
# A/B of probe options on one workload: bash tools/ab.sh <tag> <workload> "<opts1>" "<opts2>" ...
# each opts = space-separated NAME=VALUE (empty string = defaults)
T=$1; W=$2; shift 2
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in "$@"; do
  args=""; for kv in $o; do args="$args --opt $kv"; done
  for rep in 1 2; do
    timeout 600 python bench.py --workload $W --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --no-parity $args 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$W', '[$o]', f\"{d['ms_per_step']:.3f} ms  frac {d['roofline']['frac']:.3f}\", d['check'])" || echo "$W [$o] FAILED"
  done
done | tee gpurun_out/${T}_ab_${W}.txt
