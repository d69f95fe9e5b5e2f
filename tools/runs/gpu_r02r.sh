#!/bin/bash
# k_recon8 v1 + prefetched read-only O6 rows: parity, A/B vs v1
timeout 600 python -m pytest tests/test_gpu_eighttap.py -q -x > gpurun_out/t_r_8tap.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_r_8tap.log
tail -2 gpurun_out/t_r_8tap.log
LIBS="default tools/bin/lib_r8pf_minb3.so tools/bin/lib_r8v1.so default" BENCH_ARGS="--interp regular" STEPS=3 bash tools/ab_libs.sh > gpurun_out/ab_r8b.txt 2>&1
cat gpurun_out/ab_r8b.txt
