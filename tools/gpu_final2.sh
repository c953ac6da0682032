#!/bin/bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
rm -rf gpurun_out/parity gpurun_out/r2b
bash tools/gpu_round.sh r2b
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2b/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r2b/smoke.log
for C in C2a C3 C4a C4b C5 C1; do
  timeout 600 python bench.py --config $C --steps 10 > gpurun_out/r2b/bench_$C.json 2> gpurun_out/r2b/bench_$C.err; echo "$C rc=$?"
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r2b/bench_reference.json 2> gpurun_out/r2b/bench_reference.err
