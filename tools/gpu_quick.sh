#!/bin/bash
# build, GPU parity tests, batch sweep at G=8, bench without the CPU baseline
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
T=${TESTS:-tests}
timeout 1500 python -m pytest $T -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
timeout 600 python tools/batch_sweep.py C3 ${SWEEP_G:-8} 1400 > gpurun_out/sweep.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline --steps 5 > gpurun_out/bench_quick.log 2>&1
