#!/bin/bash
# Compare library variants in exp/*.so on config C2 across refill thresholds.
for v in exp/*.so; do
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  echo "== $v"; KS="${KS:-6 8 10 12 16}" bash tools/refill_sweep.sh
done
