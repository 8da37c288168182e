#!/bin/bash
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_direction.py -x -q > gpurun_out/pytest_dir.log 2>&1; echo rc=$? >> gpurun_out/pytest_dir.log
timeout 600 python tools/pull_compare.py C3 12 > gpurun_out/pull_c3.txt 2>&1
timeout 600 python tools/pull_compare.py C5 4 > gpurun_out/pull_c5.txt 2>&1
timeout 600 python tools/batch_sweep.py C3 8 1400 > gpurun_out/sweep.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline --steps 5 > gpurun_out/bench_quick.log 2>&1
