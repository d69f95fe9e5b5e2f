#!/bin/bash
# end conv (k_conv_rot EPI_RESID): residual rows through a 3-deep register queue (loop unrolled by 3):
# SR parity of the in-tree build, then base (= recon edge-permute commit) vs rq3 on one box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x -k "sr or seam or whole or c4 or i420 or ring" > gpurun_out/t_zq.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zq.log
tail -2 gpurun_out/t_zq.log
LIBS="tools/bin/lib_fixp_only.so tools/bin/lib_rq3.so tools/bin/lib_fixp_only.so tools/bin/lib_rq3.so tools/bin/lib_fixp_only.so tools/bin/lib_rq3.so" bash tools/ab_libs.sh
