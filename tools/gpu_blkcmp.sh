#!/bin/bash
OUT=gpurun_out/${1:-blkcmp}; mkdir -p $OUT
cp paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so /tmp/keep.so
for rep in 1 2; do
for v in varlib/*.so; do
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  echo "== $v"; timeout 600 python tools/large_shapes.py --schedules 5 --shapes "4,3;5,4;4,8;4,10;6,6" 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); print(d['m'], d['n'], d.get('ms'))"
done; done
cp /tmp/keep.so paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
