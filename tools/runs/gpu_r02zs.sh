#!/bin/bash
# per-shape SR batch (about two waves of the fused res-block: 49 jobs at 360p, 16 at 720p):
# full GPU suite, then c5 (512 mixed streams, one GPU) per-shape vs the old fixed 16 on one box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/t_zs.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zs.log
tail -2 gpurun_out/t_zs.log
STEPS=3 BENCH_ARGS="--config 5" LIBS="default env:NS_SR_BATCH=16 default env:NS_SR_BATCH=16" bash tools/ab_libs.sh
