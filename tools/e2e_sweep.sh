#!/bin/bash
# e2e (sshopm_run_host, pinned host buffers) per chunk size on C2
for CH in ${CHUNKS:-16384 32768 65536 131072 262144}; do
  timeout 300 python bench.py --steps 5 --no-cpu --e2e-chunk $CH > gpurun_out/e2e.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/e2e.json')); print('chunk $CH', round(d['ms_per_step'],3), 'device ms', round(d['e2e']['ms_per_step'],3), 'e2e ms')"
done
