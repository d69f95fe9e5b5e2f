#!/bin/bash
# compute-sanitizer on the c1 workload (tools/sanitize_c1.py); logs in gpurun_out/san_*.log
python -c "import __graft_entry__ as g; g.build()" || exit 1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_c1.py > gpurun_out/san_$tool.log 2>&1
  echo "$tool exit $?" >> gpurun_out/san_summary.txt
  tail -3 gpurun_out/san_$tool.log >> gpurun_out/san_summary.txt
done
