#!/bin/bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
OUT=gpurun_out/e2e4; rm -rf $OUT; mkdir -p $OUT
SSHOPM_E2E_TRACE=$OUT/trace_64k.txt timeout 300 python bench.py --steps 3 --no-cpu > $OUT/b64k.json 2>$OUT/b64k.err
python -c "import json; d=json.load(open('$OUT/b64k.json')); print('dev', round(d['ms_per_step'],3), 'e2e', round(d['e2e']['ms_per_step'],3))"
grep "host ms" $OUT/trace_64k.txt
