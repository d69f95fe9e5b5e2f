#!/bin/bash
# global selection step without host copies / syncs: NEXT-1 GPU tests, then topk vs global c4 lines on one box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_next.py tests/test_gpu_peer.py -q > gpurun_out/t_zy.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zy.log
tail -2 gpurun_out/t_zy.log
STEPS=5 LIBS="default" BENCH_ARGS="" bash tools/ab_libs.sh
STEPS=5 LIBS="default" BENCH_ARGS="--select global" bash tools/ab_libs.sh
cp gpurun_out/ab.json gpurun_out/b_zy_global.json
STEPS=5 LIBS="default" BENCH_ARGS="" bash tools/ab_libs.sh
STEPS=5 LIBS="default" BENCH_ARGS="--select global" bash tools/ab_libs.sh
