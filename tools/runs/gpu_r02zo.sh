#!/bin/bash
# the bench-configuration parity test (64 x 720p->4K streams in one call)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_c4_config.py -v > gpurun_out/t_zo.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zo.log
tail -8 gpurun_out/t_zo.log
