#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
NS_LIB=$PWD/tools/bin/lib_up_ew.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py -q -x -k "sr or seam or whole" > gpurun_out/t_z9.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_z9.log
tail -2 gpurun_out/t_z9.log
LIBS="default tools/bin/lib_up_ew.so default tools/bin/lib_up_ew.so" bash tools/ab_libs.sh
