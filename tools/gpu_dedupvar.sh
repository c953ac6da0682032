#!/bin/bash
# dedup variants: ms/step - ms solve/step = dedup time (C2)
cp paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so /tmp/keep.so
for rep in 1 2; do for v in varlib/*.so; do
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  timeout 300 python bench.py --steps 20 --no-cpu --no-e2e > /tmp/b.json 2>/dev/null
  python -c "import json; d=json.load(open('/tmp/b.json')); print('$v', round(d['ms_per_step'],4), round(d['ms_solve_per_step'],4), 'dedup+gap', round(d['ms_per_step']-d['ms_solve_per_step'],4))"
done; done
cp /tmp/keep.so paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
