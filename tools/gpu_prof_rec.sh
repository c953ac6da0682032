#!/bin/bash
# ncu --set full of the records path kernels (C2) and of the two-pass dedup, summaries via ncu_summary.py
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"sshopm_solve_rec|sshopm_dedup128" -c 2 --launch-skip 4 \
  -o gpurun_out/rec -f python tools/prof_rec.py C2 4 ${K:-4} ${U:-32} > gpurun_out/ncu_rec.log 2>&1
for k in solve_rec dedup128; do
  ncu -i gpurun_out/rec.ncu-rep -k regex:$k --page raw --csv > gpurun_out/rec_$k.csv 2>/dev/null
done
python tools/ncu_summary.py gpurun_out/rec.ncu-rep > gpurun_out/rec_summary.txt 2>&1
