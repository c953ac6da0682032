#!/bin/bash
# (4,3) solve-kernel variants in varlib/*.so on C2 (solve time, K sweep)
OUT=gpurun_out/${1:-var43}; mkdir -p $OUT
VARDIR=varlib KS="${KS:-6 8 10}" bash tools/variant_sweep.sh > $OUT/variants.txt 2>&1
cat $OUT/variants.txt
