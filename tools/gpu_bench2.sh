#!/bin/bash
# the multi-rank bench path on a one-GPU box: 2 ranks on cuda:0 over gloo (KGS_BENCH_ONE_GPU=1)
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
KGS_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --groups 2 --latency-steps 10 > gpurun_out/bench2.log 2>&1
echo rc=$? >> gpurun_out/bench2.log
