#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests/test_gpu_ring.py tests/test_gpu_host_path.py -q -x > gpurun_out/t_z3.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_z3.log; tail -4 gpurun_out/t_z3.log
