#!/bin/bash
# r02ad: C4 batch under parameter variants (prune bound, round-1 size, deferral threshold); multi-rank
# bench path on one GPU (2 ranks over gloo, groups split)
mkdir -p gpurun_out
for P in "" "prune=2" "prune_min=256" "prune_min=2048" "defer_min=16384" "defer_min=262144"; do
  PARAMS="$P" timeout 900 python tools/batch_sweep.py C4 8 >> gpurun_out/r02ad_c4_params.txt 2>&1
done
KGS_BENCH_ONE_GPU=1 timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --latency-steps 10 --no-cpu-baseline > gpurun_out/r02ad_bench_2rank.json 2> gpurun_out/r02ad_bench_2rank.err
