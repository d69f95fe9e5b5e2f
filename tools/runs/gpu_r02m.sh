#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_i420.py tests/test_gpu_host_path.py -q -x > gpurun_out/t_m_i420.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_m_i420.log
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/t_m.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_m.log
for L in tools/bin/lib_rpt12ty2.so tools/bin/lib_rpt3.so tools/bin/lib_ty8.so; do
  NS_LIB=$PWD/$L timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py -q -x -k "reconstruct" > gpurun_out/t_m_$(basename $L .so).log 2>&1; echo "rc=$?" >> gpurun_out/t_m_$(basename $L .so).log
done
LIBS="default tools/bin/lib_rpt12ty2.so tools/bin/lib_rpt3.so tools/bin/lib_ty8.so default" bash tools/ab_libs.sh > gpurun_out/ab_rpt.txt 2>&1
