#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/bin/mem_probe tools/mem_probe.cu
tools/bin/mem_probe > gpurun_out/probe.txt 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none --csv tools/bin/mem_probe > gpurun_out/probe_ncu.csv 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/t_d.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_d.log
LIBS="default tools/bin/lib_carve81.so tools/bin/lib_carve65.so tools/bin/lib_carve75.so" bash tools/ab_libs.sh > gpurun_out/ab_carve.txt 2>&1
