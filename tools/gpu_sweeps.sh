#!/bin/bash
OUT=gpurun_out/${1:-sweeps}; mkdir -p $OUT
bash tools/nsweep.sh > $OUT/nsweep.txt 2>&1; cat $OUT/nsweep.txt
timeout 1500 python tools/large_shapes.py --tensors 65536 --schedules 3,5 > $OUT/shapes64k.jsonl 2>&1; echo "rc=$?"
python -c "
import json
for l in open('$OUT/shapes64k.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['m'], d['n'], d['schedule'], d.get('ms'), d.get('alg_gflops'))"
