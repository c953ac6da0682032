#!/bin/bash
# build + run the prototype on a GPU box (cwd = repo root)
set -e
cd tools/proto_ucoef
I="-I../../include -I../../paper_conf_ipps_ballardkp11_b200/csrc"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -lineinfo $I -cubin -o uc_kern.cubin uc_kern.cu
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr $I -Xcompiler -fPIC -shared -o uc_host.so uc_host.cu -lcuda
cd ../..
mkdir -p gpurun_out
UC_NMOD=2048 UC_WIDE=4:8,1:8,8:8,4:4 UC_SETS=none python tools/proto_ucoef/run_proto.py 2>&1 | tee -a gpurun_out/proto_uc.txt
