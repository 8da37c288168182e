#!/bin/bash
# r02a: where batch time goes on C3 (G = 8, 16) — phase shares per group; then the bench as it stands
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python tools/batch_sweep.py C3 8,16 > gpurun_out/r02a_batch_c3.txt 2>&1
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r02a_bench.json 2> gpurun_out/r02a_bench.err
tail -3 gpurun_out/r02a_batch_c3.txt gpurun_out/r02a_bench.json
