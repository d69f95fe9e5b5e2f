timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/t3.log 2>&1; echo TESTS $? >> gpurun_out/t3.log
LIBS="default tools/bin/lib_out1.so default tools/bin/lib_out1.so" bash tools/ab_libs.sh > gpurun_out/ab1.txt 2>&1
