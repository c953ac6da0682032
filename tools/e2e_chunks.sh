#!/bin/bash
# e2e (run_host) chunk-size sweep: tools/e2e_chunks.sh "C2:16384,32768 C5:262144" -> gpurun_out/e2e_chunks.txt
mkdir -p gpurun_out; : > gpurun_out/e2e_chunks.txt
for spec in $1; do
  C=${spec%%:*}; for ch in $(echo ${spec#*:} | tr ',' ' '); do
    timeout 600 python bench.py --config $C --steps ${STEPS:-5} --warmup 3 --no-cpu --e2e-chunk $ch > gpurun_out/e2e_tmp.json 2> gpurun_out/e2e_tmp.err
    python - "$C" "$ch" >> gpurun_out/e2e_chunks.txt <<'PY'
import json, sys
try:
    d = json.loads(open("gpurun_out/e2e_tmp.json").read().strip().splitlines()[-1])
    print(sys.argv[1], sys.argv[2], round(d["ms_per_step"], 3), round(d["e2e"]["ms_per_step"], 3))
except Exception as e:
    print(sys.argv[1], sys.argv[2], "failed", open("gpurun_out/e2e_tmp.err").read()[-300:].replace("\n", " "))
PY
  done
done
cat gpurun_out/e2e_chunks.txt
