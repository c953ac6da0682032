#!/bin/bash
# steps-per-trip 3 and scalar-tail variants on the larger shapes (C3 (6,3), C4a (8,3), C4b (4,6))
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
OUT=gpurun_out/bigshape.jsonl; rm -f $OUT
for C in C3 C4a C4b; do
  timeout 400 python tools/solve_sweep.py --config $C --sets "1:6:0,1:8:0" >> $OUT 2>&1
  for v in gt1 st3 gt1st3; do
    [ $C = C4b ] && [ $v != st3 ] && continue
    timeout 400 env SSHOPM_LIBRARY=$PWD/variants/$v.so python tools/solve_sweep.py --config $C --sets "1:6:0,1:8:0,1:10:0" >> $OUT 2>&1
  done
done
