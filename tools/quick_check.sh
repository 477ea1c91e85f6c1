#!/bin/bash
# Quick GPU check after a kernel change: parity tests (not the full-size ones) + bench lines.
# Usage: bash tools/quick_check.sh <tag> "<workloads>"
T=${1:-q}; WLS=${2:-"c3 c5"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${T}_build.log 2>&1 || { tail -20 gpurun_out/${T}_build.log; exit 1; }
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q -p no:cacheprovider > gpurun_out/${T}_pytest.log 2>&1
echo "pytest rc=$?"; tail -4 gpurun_out/${T}_pytest.log
for w in $WLS; do
  timeout 600 python bench.py --workload $w --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --no-parity > gpurun_out/${T}_bench_$w.json 2> gpurun_out/${T}_bench_$w.err
  python - "$w" gpurun_out/${T}_bench_$w.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[2]).read().strip().splitlines()[-1])
    print(sys.argv[1], f"{d['value']:.3e} pts/s  {d['ms_per_step']:.3f} ms  frac {d['roofline']['frac']:.3f}  kern {d['roofline']['kernel_ms']:.3f} ms", d.get("check"))
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
