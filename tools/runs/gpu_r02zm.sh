#!/bin/bash
# recon per-warp residual-tile barriers (no CTA barrier): parity + A/B vs base
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "recon or whole or ring or adversarial or i420" > gpurun_out/t_zm.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zm.log
tail -2 gpurun_out/t_zm.log
LIBS="tools/bin/lib_base.so tools/bin/lib_wbar.so tools/bin/lib_base.so tools/bin/lib_wbar.so tools/bin/lib_base.so tools/bin/lib_wbar.so" bash tools/ab_libs.sh
