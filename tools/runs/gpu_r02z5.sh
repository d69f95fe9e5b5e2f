#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests/test_gpu_eighttap.py -q -x > gpurun_out/t_z5.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_z5.log; tail -2 gpurun_out/t_z5.log
LIBS="default tools/bin/lib_r8_la6.so tools/bin/lib_r8_u2.so tools/bin/lib_r8_la2.so default" BENCH_ARGS="--interp regular" STEPS=3 bash tools/ab_libs.sh
