LIBS="tools/bin/lib_up5.so tools/bin/lib_up6.so tools/bin/lib_up7.so tools/bin/lib_up5.so tools/bin/lib_up6.so tools/bin/lib_up7.so" bash tools/ab_libs.sh > gpurun_out/ab1.txt 2>&1
