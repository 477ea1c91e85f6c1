#!/bin/bash
# Round-2 bench lines of every workload (current code): full default line for C3, then the others.
T=${1:-r02m}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python bench.py > gpurun_out/${T}_bench_c3.json 2> gpurun_out/${T}_bench_c3.err; echo "c3 rc=$?"
for w in c2 c4 c5 dj dj2 knn ov pp c1; do
  timeout 900 python bench.py --workload $w --steps 20 --warmup 3 > gpurun_out/${T}_bench_$w.json 2> gpurun_out/${T}_bench_$w.err; echo "$w rc=$?"
done
for w in c3 c2 c4 c5 dj dj2 knn ov pp c1; do
  python - $w gpurun_out/${T}_bench_$w.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[2]).read().strip().splitlines()[-1])
    r = d["roofline"]; cb = d.get("cpu_baseline") or {}
    print(sys.argv[1], f"{d['value']:.3e} {d['unit']}  {d['ms_per_step']:.3f} ms  frac {r['frac']:.3f}", "cpu", f"{cb.get('value', 0):.3e}",
          "parity", (d.get("parity") or {}).get("ok"), "e2e", f"{(d.get('e2e') or {}).get('value', 0):.3e}", d.get("clocks", {}).get("reasons"))
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
