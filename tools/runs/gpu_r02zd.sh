#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/t_zd.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zd.log
tail -2 gpurun_out/t_zd.log
rm -f gpurun_out/san_summary.txt; bash tools/gpu_sanitize.sh; cat gpurun_out/san_summary.txt | grep -v "^8-tap\|^sanitize"
