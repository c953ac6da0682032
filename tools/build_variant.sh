#!/bin/bash
# Build a variant of libsshopm.so with extra nvcc flags into variants/<name>.so
# (its own object directory; the in-tree product library is never touched).
# Load it with SSHOPM_LIBRARY=variants/<name>.so (tools/solve_sweep.py --libs).
#   tools/build_variant.sh steps2 -DSSHOPM_STEPS=2
set -e
name=$1; shift
cd "$(dirname "$0")/.."
SSHOPM_BUILD_DIR=/tmp/sshopm_var_$name SSHOPM_LIB_OUT=$PWD/variants/$name.so SSHOPM_NVCC_EXTRA="$*" \
  python -m paper_conf_ipps_ballardkp11_b200.build
