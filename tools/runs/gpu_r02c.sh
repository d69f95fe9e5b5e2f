#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_ring.py tests/test_gpu_abi.py tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/t_ring.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_ring.log
timeout 900 python bench.py --config 5 --steps 3 --warmup 2 > gpurun_out/b_c5.log 2>&1
timeout 600 python bench.py --config 3 --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_c3.log 2>&1
LIBS="default tools/bin/lib_l2pf128.so tools/bin/lib_l2pf256.so tools/bin/lib_carve75.so tools/bin/lib_carve50.so" bash tools/ab_libs.sh > gpurun_out/ab_recon.txt 2>&1
for L in default tools/bin/lib_l2pf128.so tools/bin/lib_l2pf256.so tools/bin/lib_carve75.so tools/bin/lib_carve50.so; do
  if [ "$L" = default ]; then unset NS_LIB; else export NS_LIB=$PWD/$L; fi
  n=$(basename $L .so)
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k_recon_step -s 20 -c 2 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_recon_$n.csv 2>&1
done
unset NS_LIB
