#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_i420.py -q -x > gpurun_out/t_g_i420.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_g_i420.log
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/t_g.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_g.log
python bench.py --encode > gpurun_out/b_g.json 2>gpurun_out/b_g.err
