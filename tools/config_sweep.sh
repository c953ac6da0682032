#!/bin/bash
# Sweep steps-per-trip builds (exp/s<k>.so) x refill threshold K on configs C3, C4a, C4b (solve time only).
mkdir -p gpurun_out/csweep
for v in exp/*.so; do
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  for C in ${CONFIGS:-C3 C4a C4b}; do
    for K in ${KS:-6 8 10 12}; do
      timeout 300 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu --refill $K > gpurun_out/csweep/r.json 2>/dev/null
      python -c "import json; d=json.load(open('gpurun_out/csweep/r.json')); print('$(basename $v .so) $C K=$K', round(d['ms_solve_per_step'],3), 'ms solve', round(d['roofline']['frac'],3))"
    done
  done
done
