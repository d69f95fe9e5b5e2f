#!/bin/bash
# recon staging/early-barrier A/B + one ncu --set full capture of k_recon_step (source-level stalls)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "recon or whole or ring or adversarial" > gpurun_out/t_zl.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zl.log
tail -2 gpurun_out/t_zl.log
LIBS="tools/bin/lib_base.so tools/bin/lib_stage_bar.so tools/bin/lib_base.so tools/bin/lib_stage_bar.so tools/bin/lib_base.so tools/bin/lib_stage_bar.so" bash tools/ab_libs.sh
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_recon_step -s 30 -c 1 -o gpurun_out/zl_recon $B > gpurun_out/zl_recon.log 2>&1
echo "NCU rc=$?"
