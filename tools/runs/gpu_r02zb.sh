#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
NS_LIB=$PWD/tools/bin/lib_up_ldx.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_i420.py -q -x -k "sr or seam or whole" > gpurun_out/t_zb.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zb.log
tail -2 gpurun_out/t_zb.log
LIBS="default tools/bin/lib_up_ldx.so default tools/bin/lib_up_ldx.so" bash tools/ab_libs.sh
