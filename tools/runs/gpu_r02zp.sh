#!/bin/bash
# recon edge replication by selector permutes behind a warp-uniform branch (+ row-invariant clamped staging):
# parity of the in-tree build (= lib_fixp), then base / fixp_only / fixp on one box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "recon or whole or ring or adversarial or i420 or host" > gpurun_out/t_zp.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zp.log
tail -2 gpurun_out/t_zp.log
LIBS="tools/bin/lib_base.so tools/bin/lib_fixp_only.so tools/bin/lib_fixp.so tools/bin/lib_base.so tools/bin/lib_fixp_only.so tools/bin/lib_fixp.so tools/bin/lib_base.so tools/bin/lib_fixp_only.so tools/bin/lib_fixp.so" bash tools/ab_libs.sh
