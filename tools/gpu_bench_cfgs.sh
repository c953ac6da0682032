#!/bin/bash
# bench lines for selected configs + one ncu --set full capture of each config's solve kernel
OUT=gpurun_out/cfg; mkdir -p $OUT
for C in ${CFGS:-C3 C4a}; do
  timeout 600 python bench.py --config $C --steps 10 > $OUT/bench_$C.json 2> $OUT/bench_$C.err; echo "$C rc=$?"
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:sshopm_solve -s 3 -c 1 \
      -o $OUT/prof_solve_$C python bench.py --config $C --steps 1 --warmup 1 --no-e2e --no-cpu > $OUT/ncu_$C.log 2>&1; echo "ncu $C rc=$?"
  python tools/ncu_summary.py $OUT/prof_solve_$C.ncu-rep > $OUT/ncu_solve_summary_$C.txt 2>&1
done
