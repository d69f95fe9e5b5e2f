#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_i420.py -q -x > gpurun_out/t_h_i420.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_h_i420.log
NS_OVERLAP_PARTS=2 timeout 900 python -m pytest tests -m gpu -q -x -k "enhance or ring or c2_whole or host" > gpurun_out/t_h_overlap.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_h_overlap.log
LIBS="default env:NS_OVERLAP_PARTS=2 env:NS_OVERLAP_PARTS=4 default env:NS_OVERLAP_PARTS=2" bash tools/ab_libs.sh > gpurun_out/ab_overlap.txt 2>&1
python bench.py --encode > gpurun_out/b_h.json 2>gpurun_out/b_h.err
NS_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --config 5 --gpus 2 --steps 2 --warmup 1 --backend gloo > gpurun_out/b_c5_2rank.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/t_h.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_h.log
