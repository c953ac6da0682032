#!/bin/bash
# e2e pipeline timeline (SSHOPM_E2E_TRACE) and chunk-size sweep on C2
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
OUT=gpurun_out/e2e3; rm -rf $OUT; mkdir -p $OUT
SSHOPM_E2E_TRACE=$OUT/trace_64k.txt timeout 300 python bench.py --steps 3 --no-cpu > $OUT/b64k.json 2>$OUT/b64k.err
for ch in 32768 65536 131072; do for R in 0 1; do
  SSHOPM_RAMP=$R timeout 300 python bench.py --steps 10 --no-cpu --e2e-chunk $ch > $OUT/e_${ch}_$R.json 2>/dev/null
  python -c "import json; d=json.load(open('$OUT/e_${ch}_$R.json')); print('chunk $ch ramp $R dev', round(d['ms_per_step'],3), 'e2e', round(d['e2e']['ms_per_step'],3))"
done; done
SSHOPM_E2E_TRACE=$OUT/trace_32k.txt timeout 300 python bench.py --steps 3 --no-cpu --e2e-chunk 32768 > /dev/null 2>&1
