#!/bin/bash
cd "$(dirname "$0")"
mkdir -p $GRAFT_REPO_ROOT/gpurun_out
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > $GRAFT_REPO_ROOT/gpurun_out/mb_clocks.csv &
SMI=$!
./fp32_pipe | tee $GRAFT_REPO_ROOT/gpurun_out/fp32_pipe.jsonl
kill $SMI
