#!/bin/bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
rm -rf gpurun_out/parity
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
: > gpurun_out/var2.jsonl
timeout 200 python tools/solve_sweep.py --config C2 --sets "1:8:0" >> gpurun_out/var2.jsonl 2>&1
for v in raw5 raw6 smono; do
  timeout 300 env SSHOPM_LIBRARY=$PWD/variants/$v.so python tools/solve_sweep.py --config C2 --sets "1:8:0,1:6:0,1:12:0" >> gpurun_out/var2.jsonl 2>&1
done
