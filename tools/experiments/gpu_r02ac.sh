#!/bin/bash
# r02ac: determinism of the batch launch (per-query statistics and answers over repeated launches), the
# bench line with the traffic of this build, and the multi-rank bench path on one GPU (2 ranks over gloo)
mkdir -p gpurun_out
timeout 900 python tools/determinism_check.py C4 3 8 > gpurun_out/r02ac_determinism_c4.txt 2>&1
timeout 600 python tools/determinism_check.py C3 3 8 > gpurun_out/r02ac_determinism_c3.txt 2>&1
timeout 1200 python bench.py > gpurun_out/r02ac_bench.json 2> gpurun_out/r02ac_bench.err
KGS_BENCH_ONE_GPU=1 timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --latency-steps 10 --no-cpu-baseline > gpurun_out/r02ac_bench_2rank.json 2> gpurun_out/r02ac_bench_2rank.err
