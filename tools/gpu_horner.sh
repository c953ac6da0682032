#!/bin/bash
# n = 3 Horner variant (SSHOPM_HORNER3): C3 / C4a solve times vs the product build, parity tests on the variant
mkdir -p gpurun_out
for C in C3 C4a; do
  CFG=$C REPS=5 bash tools/gpu_var.sh "1:0:0,1:6:0,1:4:0" paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so,variants/${VAR:-horner3}.so
done
SSHOPM_LIBRARY=$PWD/variants/${VAR:-horner3}.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -x -q -k "6-3 or 8-3 or 5-3 or C3 or C4a or shapes or fixed_k" 2>&1 | tail -4 | tee gpurun_out/horner_tests.txt
