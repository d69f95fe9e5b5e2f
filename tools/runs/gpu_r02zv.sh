#!/bin/bash
# final HEAD check: full GPU suite + smoke
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/t_zv.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zv.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_zv.log 2>&1; echo "SMOKE rc=$?" >> gpurun_out/smoke_zv.log
tail -2 gpurun_out/t_zv.log; tail -2 gpurun_out/smoke_zv.log
