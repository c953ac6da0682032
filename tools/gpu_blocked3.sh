#!/bin/bash
OUT=gpurun_out/${1:-blk3}; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:randomly --timeout 300 -k "blocked or general" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
tail -3 $OUT/pytest.log
timeout 900 python tools/large_shapes.py --schedules 5 > $OUT/shapes5.jsonl 2>&1; echo "rc=$?"
cat $OUT/shapes5.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sshopm_blocked -s 1 -c 1 -o $OUT/prof_blocked \
  python tools/large_shapes.py --shapes "4,10" --schedules 5 > $OUT/ncu.log 2>&1; echo "ncu rc=$?"
