#!/bin/bash
# Blocked-kernel session: its GPU tests, the general-kernel tests, and the large-shape timing table.
OUT=gpurun_out/${1:-blk}; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:randomly --timeout 300 -k "blocked or general" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
tail -15 $OUT/pytest.log
timeout 900 python tools/large_shapes.py > $OUT/large_shapes.jsonl 2> $OUT/large_shapes.err; echo "large rc=$?"
cat $OUT/large_shapes.jsonl; tail -3 $OUT/large_shapes.err
