#!/bin/bash
# compute-sanitizer evidence (VERDICT r1 Next 6): memcheck / racecheck / synccheck / initcheck on small runs.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out/sanitizer
timeout 600 python -m pytest tests -x -q -m gpu -k "schedule7 or records_only or plain_sshopm or fused_vs_oracle" > gpurun_out/pytest_new.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_new.log
for c in ${CASES:-two_pass lean tpl wt wt_records fused blocked general classify run_host}; do
  for tool in memcheck racecheck synccheck initcheck; do
    timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py $c \
      > gpurun_out/sanitizer/${c}_${tool}.log 2>&1
    echo "$c $tool rc=$?" >> gpurun_out/sanitizer/summary.txt
  done
done
