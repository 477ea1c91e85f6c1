#!/bin/bash
# GPU-box check: parity tests + bench lines of every workload.  Usage: bash tools/gpu_check.sh <tag>
T=${1:-chk}
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_pytest.log 2>&1; tail -3 gpurun_out/${T}_pytest.log
WLS="${WLS:-c3 c2 c4 c5 dj dj2 knn ov}" STEPS=${STEPS:-20} bash tools/bench_matrix.sh > gpurun_out/${T}_matrix.txt 2>&1
cat gpurun_out/${T}_matrix.txt
