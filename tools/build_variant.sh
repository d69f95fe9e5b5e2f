#!/bin/bash
# Build libneuroscaler with extra defines into tools/bin/$OUT (A/B timing: NS_LIB=tools/bin/$OUT python bench.py)
set -e
cd "$(dirname "$0")/.."
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -I include"
T=$(mktemp -d)
for s in ns_api k_select k_recon k_sr ns_hybrid; do
  nvcc $F $EXTRA -c paper_conf_sigcomm_yeolkjyh22_b200/csrc/$s.cu -o $T/$s.o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o tools/bin/$OUT $T/*.o -lcudart_static -lnvjpeg
rm -rf $T
