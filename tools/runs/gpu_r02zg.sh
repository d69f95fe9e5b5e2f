#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/t_zg.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zg.log
tail -2 gpurun_out/t_zg.log
timeout 300 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_c1.py > gpurun_out/san_racecheck_zg.log 2>&1; tail -2 gpurun_out/san_racecheck_zg.log
timeout 300 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_c1.py > gpurun_out/san_memcheck_zg.log 2>&1; tail -2 gpurun_out/san_memcheck_zg.log
timeout 300 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_c1.py > gpurun_out/san_synccheck_zg.log 2>&1; tail -2 gpurun_out/san_synccheck_zg.log
