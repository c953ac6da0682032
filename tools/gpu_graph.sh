#!/bin/bash
OUT=gpurun_out/${1:-graph}; mkdir -p $OUT
for L in 10 12 14 16 20; do for G in "" "--graph"; do
  N=$((1 << L))
  timeout 300 python bench.py --voxels $N --steps 20 --no-cpu --no-e2e $G > $OUT/n${L}${G}.json 2> $OUT/n${L}${G}.err
  python -c "import json; d=json.load(open('$OUT/n${L}${G}.json')); print('2^$L', '$G', round(d['ms_per_step'],4), 'ms/step', d['gpu_launches'], 'launches', d['config']['cuda_graph'])" 2>&1 | tail -1
done; done
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "C1_full" 2>&1 | tail -1
