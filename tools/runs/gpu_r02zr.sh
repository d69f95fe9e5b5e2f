#!/bin/bash
# k_conv_rot warp-specialised (MMA warp + 4 epilogue warps, E(q) releases the block before its stores) + 3-deep residual queue:
# SR parity of the in-tree build, then base (= recon edge-permute commit) vs rq3 on one box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x -k "sr or seam or whole or c4 or i420 or ring" > gpurun_out/t_zr.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zr.log
tail -2 gpurun_out/t_zr.log
LIBS="tools/bin/lib_fixp_only.so tools/bin/lib_ws.so tools/bin/lib_fixp_only.so tools/bin/lib_ws.so tools/bin/lib_fixp_only.so tools/bin/lib_ws.so" bash tools/ab_libs.sh
