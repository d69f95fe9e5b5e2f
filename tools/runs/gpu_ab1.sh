timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/t3.log 2>&1; echo TESTS $? >> gpurun_out/t3.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo SMOKE $? >> gpurun_out/smoke.log
python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/last_bench.json 2>&1
