#!/bin/bash
OUT=gpurun_out/${1:-e2e2}; mkdir -p $OUT
for rep in 1 2; do for R in 0 1; do for ch in 32768 65536; do
  SSHOPM_RAMP=$R timeout 300 python bench.py --steps 20 --no-cpu --e2e-chunk $ch > $OUT/e2e_${R}_${ch}_$rep.json 2>/dev/null
  python -c "import json; d=json.load(open('$OUT/e2e_${R}_${ch}_$rep.json')); print('ramp $R chunk $ch', round(d['ms_per_step'],3), 'dev', round(d['e2e']['ms_per_step'],3), 'e2e')"
done; done; done
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:randomly -k run_host 2>&1 | tail -2
