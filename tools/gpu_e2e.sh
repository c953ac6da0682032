#!/bin/bash
OUT=gpurun_out/${1:-e2e}; mkdir -p $OUT
python tools/link_bw.py > $OUT/link_bw.json 2>&1; cat $OUT/link_bw.json
for ch in 32768 65536 131072; do
  timeout 300 python bench.py --steps 10 --no-cpu --e2e-chunk $ch > $OUT/e2e_$ch.json 2>/dev/null
  python -c "import json; d=json.load(open('$OUT/e2e_$ch.json')); print('chunk $ch', round(d['ms_per_step'],3), 'device', d['e2e'])"
done
timeout 300 python bench.py --steps 10 --no-cpu --e2e-rep > $OUT/e2e_rep.json 2>/dev/null
python -c "import json; d=json.load(open('$OUT/e2e_rep.json')); print('with rep', round(d['ms_per_step'],3), 'device', d['e2e'])"
