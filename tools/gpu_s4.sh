#!/bin/bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
tools/microbench/pipe_mix > gpurun_out/pipe_mix2.jsonl 2>&1
: > gpurun_out/cmp4.jsonl
timeout 200 python tools/solve_sweep.py --config C2 --sets "1:8:0" >> gpurun_out/cmp4.jsonl 2>&1
timeout 200 env SSHOPM_LIBRARY=$PWD/variants/f4.so python tools/solve_sweep.py --config C2 --sets "1:8:0,1:6:0,1:10:0" >> gpurun_out/cmp4.jsonl 2>&1
