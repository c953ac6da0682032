#!/bin/bash
# ncu --set full of the solve kernel: lean (schedule 1) vs round-1 refill (schedule 6), C2.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for sc in ${SCHEDS:-1 6}; do
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:sshopm_solve -c 1 --launch-skip 2 \
    -o gpurun_out/solve_s$sc -f python tools/prof_solve.py C2 $sc 3 > gpurun_out/ncu_s$sc.log 2>&1
done
timeout 300 python tools/solve_sweep.py --config C2 --sets "${SETS:-1:6:0,6:8:0,1:8:0}" > gpurun_out/sweep_cmp.jsonl 2>&1
