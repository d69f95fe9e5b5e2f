#!/bin/bash
# Round-end evidence on one GPU: all GPU tests, the default bench line, a
# --select global bench line, the launch list and ncu --set full captures.
python -m pytest tests -m gpu -x -q > gpurun_out/final_tests.log 2>&1; echo TESTS $? >> gpurun_out/final_tests.log
python bench.py > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err
python bench.py --select global --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/final_bench_global.json 2>&1
TAG=${TAG:-r01h} bash tools/profile_round.sh > gpurun_out/prof.log 2>&1
