#!/bin/bash
# one ncu --set full capture of the solve kernel per config (C3, C4a, C4b, C2a)
OUT=gpurun_out/${1:-ncucfg}; mkdir -p $OUT
for C in C2a C3 C4a C4b; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:sshopm_solve -s 3 -c 1 \
      -o $OUT/prof_solve_$C python bench.py --config $C --steps 1 --warmup 1 --no-e2e --no-cpu > $OUT/ncu_$C.log 2>&1; echo "$C rc=$?"
done
