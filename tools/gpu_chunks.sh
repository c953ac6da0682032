#!/bin/bash
# item-granular schedule-1 chunks: C1 / C2 bench lines + the tests that exercise chunking and C1 parity
mkdir -p gpurun_out/chk
for C in C1 C2; do timeout 600 python bench.py --config $C --steps 20 --no-cpu > gpurun_out/chk/bench_$C.json 2> gpurun_out/chk/bench_$C.err; echo "$C rc=$?"; done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_wide.py tests/test_gpu_fullsize.py -m gpu -q -x -k "C1 or tiny or invariance or empty or total_iters or special or wide or fixed_k or shapes or per_tensor or fused or records" 2>&1 | tail -3
