#!/bin/bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
OUT=gpurun_out/gt; rm -rf $OUT gpurun_out/parity; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
for C in C3 C2; do timeout 600 python bench.py --config $C --steps 10 --no-cpu > $OUT/bench_$C.json 2> $OUT/bench_$C.err; done
