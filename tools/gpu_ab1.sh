timeout 900 python -m pytest tests/test_gpu_next.py -x -q > gpurun_out/t3.log 2>&1; echo TESTS $? >> gpurun_out/t3.log
python bench.py --select global --balance --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bal.json 2>&1
