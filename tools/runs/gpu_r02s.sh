#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python tools/sanitize_c1.py > gpurun_out/san_plain.log 2>&1; echo "plain rc=$?" >> gpurun_out/san_plain.log
tail -12 gpurun_out/san_plain.log
rm -f gpurun_out/san_summary.txt
bash tools/gpu_sanitize.sh
cat gpurun_out/san_summary.txt
