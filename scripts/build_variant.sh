#!/bin/bash
# build an alternative libve into build/libve_$1.so with extra nvcc flags "$2" (A/B experiments)
cd "$(dirname "$0")/.." && mkdir -p build
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xptxas -O3 \
  -I include $2 -shared -o build/libve_$1.so paper_conf_asplos_zhouhmm022_b200/csrc/*.cu -ldl
