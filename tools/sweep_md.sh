#!/bin/bash
# canvas max_dim sweep: bash tools/sweep_md.sh <tag> <workload> "<max_dims>" [extra bench args]
T=$1; W=$2; MDS=$3; shift 3
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for md in $MDS; do
  timeout 600 python bench.py --workload $W --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --no-parity --max-dim $md "$@" 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); c=d['config']['canvas']; print('$W', 'max_dim $md', f\"{d['ms_per_step']:.3f} ms frac {d['roofline']['frac']:.3f}\", 'W', c['W'], 'mixed', round(c['mixed_tile_frac'],3), 'recs', c['num_records'], 'stages', {k[:8]: round(v,3) for k,v in (d.get('stages_ms') or {}).items()})" || echo "$W $md FAILED"
done | tee gpurun_out/${T}_sweep_${W}.txt
