#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x -rs --durations=15 > gpurun_out/t.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t.log
rm -f gpurun_out/san_summary.txt
bash tools/gpu_sanitize.sh
python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/b1.log 2>&1
