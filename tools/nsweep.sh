#!/bin/bash
# Fig. 5 analogue: throughput vs number of tensors, (4,3), 128 starts, alpha = 0.
mkdir -p gpurun_out/nsweep
for L in 10 12 14 16 18 20 21 22 23; do
  N=$((1 << L))
  ST=$(( L >= 22 ? 5 : 20 ))
  timeout 600 python bench.py --voxels $N --steps $ST --warmup 3 --no-cpu --no-e2e > gpurun_out/nsweep/n$L.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/nsweep/n$L.json')); print('2^$L', $N, round(d['ms_per_step'],4), round(d['ms_solve_per_step'],4), round(d['value']/1e3,2), '%.3e' % d['voxel_solves_per_s'], round(d['roofline']['frac'],3))"
done
