#!/bin/bash
# 8-tap MC: parity tests, then the recon parity suites (bilinear unaffected)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_eighttap.py -q -x > gpurun_out/t_o_8tap.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_o_8tap.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_i420.py tests/test_gpu_ring.py -q -x -k "reconstruct or ring or whole" > gpurun_out/t_o_recon.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_o_recon.log
tail -5 gpurun_out/t_o_8tap.log; tail -3 gpurun_out/t_o_recon.log
