LIBS="default tools/bin/lib_nh5.so tools/bin/lib_nh7.so default tools/bin/lib_nh5.so tools/bin/lib_nh7.so" bash tools/ab_libs.sh > gpurun_out/ab1.txt 2>&1
python tools/rb_trace2.py > gpurun_out/trace3.txt 2>&1
