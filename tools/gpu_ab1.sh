timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "two_sr_batches or enhance" > gpurun_out/t3.log 2>&1; echo TESTS $? >> gpurun_out/t3.log
