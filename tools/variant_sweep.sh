#!/bin/bash
# Compare library variants in exp/*.so on config C2 across refill thresholds.
# KS_<name> overrides the K list for exp/<name>.so.
for v in ${VARDIR:-exp}/*.so; do
  name=$(basename $v .so)
  cp $v paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so
  ks_var="KS_$name"; ks="${!ks_var:-${KS:-6 8 10 12 16}}"
  echo "== $v"; KS="$ks" bash tools/refill_sweep.sh
done
