#!/bin/bash
# peer-memory transport for moved anchors: 2-rank test on one GPU + a 2-rank bench (gloo, shared GPU)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_peer.py -q -x > gpurun_out/t_t_peer.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_t_peer.log
tail -3 gpurun_out/t_t_peer.log
for T in peer nccl; do
NS_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
  bench.py --gpus 2 --backend gloo --select global --balance --transport $T --streams 16 --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 \
  > gpurun_out/bench_t_$T.json 2> gpurun_out/bench_t_$T.err
echo "bench $T rc=$?"; tail -c 600 gpurun_out/bench_t_$T.json; tail -3 gpurun_out/bench_t_$T.err
done
