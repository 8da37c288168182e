#!/bin/bash
mkdir -p gpurun_out
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02s_pb8.log 2>&1
timeout 900 python tools/batch_sweep.py C3 8 > gpurun_out/r02s_sweep.txt 2>&1
