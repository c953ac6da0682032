#!/bin/bash
# One gpurun session: GPU tests, then solve-kernel sweeps (tools/solve_sweep.py).
#   gpurun --timeout 2400 -- bash tools/gpu_session.sh [tests|notests]
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
if [ "${1:-tests}" = "tests" ]; then
  timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
fi
S1=${SETS1:-"1:4:0,1:2:0,1:3:0,1:5:0,1:6:0,1:8:0,1:4:2,1:4:4,6:8:0"}
timeout 600 python tools/solve_sweep.py --config C2 --sets "$S1" > gpurun_out/sweep_main.jsonl 2>&1
for v in ${VARIANTS:-f43x steps2 steps4}; do
  timeout 300 env SSHOPM_LIBRARY=$PWD/variants/$v.so python tools/solve_sweep.py --config C2 --sets "${SETSV:-1:3:0,1:4:0,1:6:0}" > gpurun_out/sweep_$v.jsonl 2>&1
done
