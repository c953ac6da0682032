#!/bin/bash
cp paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so /tmp/keep.so
for rep in 1 2 3; do
for v in varlib/*.so; do
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  echo "== $v $(timeout 600 python tools/large_shapes.py --tensors 65536 --schedules 5 --shapes "5,4;4,8;5,6;6,6;4,10" 2>&1 | python -c "
import sys, json
print(' '.join(f\"{d['m']}{d['n']}:{d['ms']}\" for d in (json.loads(l) for l in sys.stdin if l.startswith('{'))))")"
done; done
cp /tmp/keep.so paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
