LIBS="default tools/bin/lib_ty8.so tools/bin/lib_tx16ty8.so default tools/bin/lib_ty8.so tools/bin/lib_tx16ty8.so" bash tools/ab_libs.sh > gpurun_out/ab1.txt 2>&1
