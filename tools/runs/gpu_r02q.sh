#!/bin/bash
# k_recon8 v2 (8-row rolled loop): parity, then A/B of register budgets and the v1 full unroll
timeout 600 python -m pytest tests/test_gpu_eighttap.py -q -x > gpurun_out/t_q_8tap.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_q_8tap.log
tail -2 gpurun_out/t_q_8tap.log
LIBS="default tools/bin/lib_r8minb3.so tools/bin/lib_r8minb4.so tools/bin/lib_r8v1.so" BENCH_ARGS="--interp regular" STEPS=3 bash tools/ab_libs.sh > gpurun_out/ab_r8.txt 2>&1
cat gpurun_out/ab_r8.txt
