python -m pytest tests/test_gpu_next.py tests/test_abi.py -x -q > gpurun_out/t2.log 2>&1; echo TESTS $? >> gpurun_out/t2.log
python tools/selector_study.py --out gpurun_out/r01_selector_study.json > gpurun_out/sel.log 2>&1
