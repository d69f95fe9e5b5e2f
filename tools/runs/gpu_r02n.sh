#!/bin/bash
# invisible frames + full GPU suite + smoke + default bench
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_next.py -q -x -k invisible > gpurun_out/t_n_inv.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_n_inv.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/t_n.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_n.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/smoke_n.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_n.json 2> gpurun_out/bench_n.err
tail -3 gpurun_out/t_n_inv.log gpurun_out/t_n.log gpurun_out/smoke_n.log; cat gpurun_out/bench_n.json
