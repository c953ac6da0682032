#!/bin/bash
# Sweep the refill threshold K on config C2 (solve time only, no e2e / cpu baseline).
mkdir -p gpurun_out/sweep
for K in ${KS:-2 4 6 8 10 12 16}; do
  timeout 200 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --refill $K "$@" > gpurun_out/sweep/k$K.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/sweep/k$K.json')); print('K=$K', round(d['ms_solve_per_step'],3), 'ms solve', round(d['roofline']['frac'],3))"
done
