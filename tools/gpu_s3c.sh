#!/bin/bash
OUT=gpurun_out/${1:-s3c}; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q -p no:randomly --timeout 300 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 900 python tools/large_shapes.py --schedules 5 > $OUT/shapes5.jsonl 2>&1; echo "rc=$?"
cat $OUT/shapes5.jsonl
