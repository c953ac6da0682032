#!/bin/bash
# full GPU test suite + C3 / C4a solve sweeps on the product build
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -p no:randomly --timeout 240 > gpurun_out/pytest_gpu_check.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_check.log
tail -4 gpurun_out/pytest_gpu_check.log
for C in ${CFGS:-C3 C4a}; do python tools/solve_sweep.py --config $C --sets "1:0:0,1:6:0,1:8:0" --reps 5 --no-total 2>&1 | grep -v Warn; done | tee gpurun_out/check_sweep.jsonl
