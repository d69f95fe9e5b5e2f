#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
NS_LIB=$PWD/tools/bin/lib_r8rolled.so timeout 900 python -m pytest tests/test_gpu_eighttap.py -q -x > gpurun_out/t_z4.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_z4.log; tail -3 gpurun_out/t_z4.log
LIBS="default tools/bin/lib_r8rolled.so default tools/bin/lib_r8rolled.so" BENCH_ARGS="--interp regular" STEPS=3 bash tools/ab_libs.sh
