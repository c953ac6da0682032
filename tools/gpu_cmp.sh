#!/bin/bash
# Compare library builds on C2 (tools/solve_sweep.py): round-1 library vs step forms x refill schedules.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
: > gpurun_out/cmp.jsonl
timeout 200 env SSHOPM_LIBRARY=$PWD/variants/r1.so python tools/solve_sweep.py --config C2 --sets "1:8:0" >> gpurun_out/cmp.jsonl 2>&1
timeout 300 env SSHOPM_LIBRARY=$PWD/variants/f43r1.so python tools/solve_sweep.py --config C2 --sets "6:8:0,1:8:0,1:6:0,1:4:0" >> gpurun_out/cmp.jsonl 2>&1
timeout 200 env SSHOPM_LIBRARY=$PWD/variants/f43x.so python tools/solve_sweep.py --config C2 --sets "6:8:0,1:6:0" >> gpurun_out/cmp.jsonl 2>&1
timeout 200 python tools/solve_sweep.py --config C2 --sets "6:8:0,1:6:0" >> gpurun_out/cmp.jsonl 2>&1
timeout 200 env SSHOPM_LIBRARY=$PWD/variants/r1.so python tools/solve_sweep.py --config C2 --sets "1:8:0" >> gpurun_out/cmp.jsonl 2>&1
