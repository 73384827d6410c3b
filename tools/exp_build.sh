#!/bin/bash
# build experiment variants of libabacus.so into exp/<name>.so: exp_build.sh name "-DFLAG ..."
cd /root/repo/paper_conf_sc_cui0czlzsmylg21_b200/csrc
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC -shared $2 \
  -o /root/repo/exp/$1.so abacus.cu kernels_simt.cu kernels_tc.cu kernels_train.cu -ldl
