#!/bin/bash
TAG=${TAG:-r2}
# Bench lines for every config (C2 default first) + C2 launch list and solve-kernel ncu capture.
OUT=gpurun_out/${1:-cfg}; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/smi.txt 2>&1
timeout 420 python bench.py > $OUT/bench_C2.json 2> $OUT/bench_C2.err; echo "C2 rc=$?"
for C in C2a C3 C4a C4b C5; do
  timeout 600 python bench.py --config $C --steps 10 > $OUT/bench_$C.json 2> $OUT/bench_$C.err; echo "$C rc=$?"
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $OUT/bench_reference.json 2> $OUT/bench_reference.err; echo "ref rc=$?"
timeout 420 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > $OUT/ncu_launch_bench.log 2>&1; echo "ncu launches rc=$?"
for f in $OUT/bench_*.json; do python -c "
import json,sys; d=json.loads(open('$f').read().splitlines()[-1]); r=d.get('roofline') or {}
print('$f', round(d.get('ms_per_step',0),3), 'ms', round(d['value'],1), d['unit'], 'frac', r.get('frac'), 'exec', r.get('executed_frac_ncu'), 'conv', d.get('converged_frac'), 'e2e', (d.get('e2e') or {}).get('ms_per_step'))" 2>&1 | tail -1; done
