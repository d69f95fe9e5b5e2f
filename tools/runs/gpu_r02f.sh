#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x -rs -s -k "hybrid or h26x or c2_whole or c3_whole or seam" > gpurun_out/t_f_print.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/t_f.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_f.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_f.log 2>&1; echo "SMOKE rc=$?" >> gpurun_out/smoke_f.log
rm -f gpurun_out/san_summary.txt; bash tools/gpu_sanitize.sh
python bench.py --encode > gpurun_out/b_f.json 2>gpurun_out/b_f.err
TAG=r02f bash tools/profile_round.sh > gpurun_out/prof_r02f.log 2>&1
