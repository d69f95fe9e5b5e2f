#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_i420.py tests/test_gpu_abi.py tests/test_gpu_host_path.py -q -x > gpurun_out/t_zc.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zc.log
tail -2 gpurun_out/t_zc.log
LIBS="default tools/bin/lib_up_old.so default tools/bin/lib_up_old.so" bash tools/ab_libs.sh
