python -m pytest tests/test_gpu_parity.py -x -q -k "sr_ or enhance" > gpurun_out/t3.log 2>&1; echo TESTS $? >> gpurun_out/t3.log
LIBS="default tools/bin/lib_nobias.so default tools/bin/lib_nobias.so" bash tools/ab_libs.sh > gpurun_out/ab1.txt 2>&1
