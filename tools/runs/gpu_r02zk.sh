#!/bin/bash
# recon word-loader / early-barrier A/B: parity of the new default build, then base vs variants on one box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x -k "recon or whole or ring or adversarial or i420 or host" > gpurun_out/t_zk.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zk.log
tail -2 gpurun_out/t_zk.log
LIBS=${LIBS:-"tools/bin/lib_base.so tools/bin/lib_words.so tools/bin/lib_words_bar.so tools/bin/lib_base.so tools/bin/lib_words.so tools/bin/lib_words_bar.so"} bash tools/ab_libs.sh
