#!/bin/bash
# One GPU session: tests, bench, ncu launch list, ncu full capture of the solve kernel.
# Usage: bash tools/gpu_round.sh <tag> [bench args...]   (env: SKIP_TESTS, SKIP_NCU, TESTS=<pytest selector>)
set -u
TAG=${1:-r1}; shift || true
OUT=gpurun_out/$TAG; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/smi.txt 2>&1
if [ -z "${SKIP_TESTS:-}" ]; then
  timeout 900 python -m pytest ${TESTS:-tests} -m gpu -q -p no:randomly --timeout 240 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
  tail -3 $OUT/pytest_gpu.log
fi
timeout 420 python bench.py "$@" > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
if [ -z "${SKIP_NCU:-}" ]; then
  timeout 420 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
      python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu "$@" > $OUT/ncu_launch_bench.log 2>&1; echo "ncu launches rc=$?"
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:sshopm_solve -s 3 -c 1 \
      -o $OUT/prof_solve python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:sshopm_dedup -s 3 -c 1 \
      -o $OUT/prof_dedup python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > $OUT/ncu_dedup.log 2>&1; echo "ncu dedup rc=$?"
fi
