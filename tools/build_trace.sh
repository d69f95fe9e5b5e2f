#!/bin/bash
# Debug timeline build (clock64 trace of CTA (0,0,0), -DNS_TRACE): tools/bin/libneuroscaler_trace.so
# Extra defines via EXTRA, e.g. EXTRA=-DNS_TRACE_NOEPI OUT=lib_trace_noepi.so tools/build_trace.sh
set -e
cd "$(dirname "$0")/.."
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -I include"
T=$(mktemp -d)
for s in ns_api k_select k_recon k_sr ns_hybrid; do
  nvcc $F -DNS_TRACE $EXTRA -c paper_conf_sigcomm_yeolkjyh22_b200/csrc/$s.cu -o $T/$s.o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o tools/bin/${OUT:-libneuroscaler_trace.so} $T/*.o -lcudart_static -lnvjpeg
rm -rf $T
