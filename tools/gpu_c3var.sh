#!/bin/bash
OUT=gpurun_out/${1:-c3var}; mkdir -p $OUT
cp paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so /tmp/keep.so
for v in varlib/*.so; do
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  for K in 6 8; do
    timeout 200 python bench.py --config C3 --steps 5 --warmup 3 --no-e2e --no-cpu --refill $K > $OUT/$(basename $v .so)_k$K.json 2>/dev/null
    python -c "import json; d=json.load(open('$OUT/$(basename $v .so)_k$K.json')); print('$v K=$K', round(d['ms_solve_per_step'],3), 'ms solve', round(d['roofline']['frac'],3))"
  done
done
cp /tmp/keep.so paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
