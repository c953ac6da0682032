#!/bin/bash
OUT=gpurun_out/${1:-blk2}; mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:randomly --timeout 300 -k "blocked" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
tail -3 $OUT/pytest.log
timeout 600 python tools/large_shapes.py --schedules 3,5 --shapes "4,3;5,4;6,4;3,6;4,5;7,3" > $OUT/small_shapes.jsonl 2>&1; echo "small rc=$?"
cat $OUT/small_shapes.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sshopm_blocked -s 1 -c 1 -o $OUT/prof_blocked \
  python tools/large_shapes.py --shapes "4,10" --schedules 5 > $OUT/ncu.log 2>&1; echo "ncu rc=$?"
