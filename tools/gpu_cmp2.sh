#!/bin/bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
: > gpurun_out/cmp2.jsonl
for rep in 1 2; do
timeout 200 python tools/solve_sweep.py --config C2 --sets "1:8:0,1:6:0,1:10:0" >> gpurun_out/cmp2.jsonl 2>&1
timeout 200 env SSHOPM_LIBRARY=$PWD/variants/f3.so python tools/solve_sweep.py --config C2 --sets "1:8:0,1:6:0,1:10:0" >> gpurun_out/cmp2.jsonl 2>&1
done
