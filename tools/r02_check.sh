#!/bin/bash
# Round-2 GPU check: build, GPU tests, default bench line (with the parity verdict), sanitizers.
# Usage (on the box): bash tools/r02_check.sh <tag> [skip_tests]
T=${1:-r02}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${T}_build.log 2>&1 || { tail -20 gpurun_out/${T}_build.log; exit 1; }
if [ -z "$2" ]; then
  timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/${T}_pytest.log 2>&1
  echo "pytest rc=$?"; tail -5 gpurun_out/${T}_pytest.log
fi
timeout 900 python bench.py > gpurun_out/${T}_bench_c3.json 2> gpurun_out/${T}_bench_c3.err
echo "bench rc=$?"; tail -c 1500 gpurun_out/${T}_bench_c3.json
for tool in memcheck racecheck synccheck; do
  q=""; [ "$tool" != "memcheck" ] && q="--quick"
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_cases.py $q \
     > gpurun_out/${T}_sanitize_${tool}.log 2>&1
  echo "sanitize $tool rc=$?"; tail -3 gpurun_out/${T}_sanitize_${tool}.log
done
