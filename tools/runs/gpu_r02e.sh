#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
K="reconstruct or enhance or c2_ or ring or host"
timeout 900 python -m pytest tests -m gpu -q -x -k "$K" > gpurun_out/t_e_default.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_e_default.log
NS_LIB=$PWD/tools/bin/lib_xlane.so timeout 900 python -m pytest tests -m gpu -q -x -k "$K" > gpurun_out/t_e_xlane.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_e_xlane.log
LIBS="default tools/bin/lib_xlane.so tools/bin/lib_carve81.so default" bash tools/ab_libs.sh > gpurun_out/ab_e.txt 2>&1
for L in default tools/bin/lib_xlane.so tools/bin/lib_carve81.so; do
  if [ "$L" = default ]; then unset NS_LIB; else export NS_LIB=$PWD/$L; fi
  n=$(basename $L .so)
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k_recon_step -s 20 -c 2 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_e_$n.csv 2>&1
done
