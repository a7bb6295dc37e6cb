#!/bin/bash
# build a libxbfs.so variant with extra nvcc defines: tools/build_variant.sh out.so [-DNAME=V ...]
out=$1; shift
nvcc -O3 -std=c++17 -lineinfo -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC,-O3 -shared -DXBFS_ARCH=100 \
  -I include "$@" paper_conf_sc_yangls0w24_b200/csrc/*.cu -o "$out"
