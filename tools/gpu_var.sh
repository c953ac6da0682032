#!/bin/bash
# A/B of variant builds on C2: tools/gpu_var.sh "<sets>" lib1,lib2,...
mkdir -p gpurun_out
python tools/solve_sweep.py --config ${CFG:-C2} --sets "$1" --libs "$2" --reps ${REPS:-7} --no-total 2>&1 | tee -a gpurun_out/var_sweep.jsonl
