#!/bin/bash
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
timeout 600 python tools/pull_compare.py C5 4 > gpurun_out/pull_c5.txt 2>&1
