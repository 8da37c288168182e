#!/bin/bash
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 900 python tools/exp_sweeps.py 30 > gpurun_out/exp_sweeps.txt 2>&1
