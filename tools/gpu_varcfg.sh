#!/bin/bash
# varlib/*.so on several configs: solve ms per step at the library-default refill threshold (2 reps)
cp paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so /tmp/keep.so
for C in ${CFGS:-C2 C3}; do for rep in 1 2; do for v in varlib/*.so; do
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  timeout 300 python bench.py --config $C --steps 10 --warmup 3 --no-e2e --no-cpu > /tmp/v.json 2>/dev/null
  python -c "import json; d=json.load(open('/tmp/v.json')); print('$C', '$v', round(d['ms_solve_per_step'],3), 'ms solve', round(d['roofline']['frac'],4))"
done; done; done
cp /tmp/keep.so paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
