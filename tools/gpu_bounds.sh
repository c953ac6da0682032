#!/bin/bash
# Debug build with device asserts on the refill / record index paths (SSHOPM_BOUNDS_CHECK; compute-sanitizer is
# closed on this pool): run the GPU tests of the records path, item chunks, Horner shapes and shift modes on it.
mkdir -p gpurun_out
SSHOPM_LIBRARY=$PWD/variants/bounds.so timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_wide.py \
  -m gpu -q -k "records or small_problem or tiny or C1 or 6-3 or 8-3 or 4-6 or per_tensor or auto_shift or invariance or wide or fixed_k or special" \
  2>&1 | tail -3 | tee gpurun_out/bounds_tests.txt
