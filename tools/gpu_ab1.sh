LIBS="default tools/bin/lib_one.so default tools/bin/lib_one.so" bash tools/ab_libs.sh > gpurun_out/ab1.txt 2>&1
