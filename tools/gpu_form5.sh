#!/bin/bash
# form-5 (Horner) variant: C2 solve time vs the product build, and the (4,3) parity tests on the variant
mkdir -p gpurun_out
python tools/solve_sweep.py --config C2 --sets "1:0:0" --libs paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so,variants/form5.so --reps 7 --no-total 2>&1 | tee gpurun_out/form5_sweep.jsonl
python tools/solve_sweep.py --config C2a --sets "1:0:0" --libs paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so,variants/form5.so --reps 5 --no-total 2>&1 | tee -a gpurun_out/form5_sweep.jsonl
SSHOPM_LIBRARY=$PWD/variants/form5.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "C1_full or fixed_k or apply or special or invariance or per_tensor or auto_shift or dedup_end" 2>&1 | tail -5 | tee gpurun_out/form5_tests.txt
