#!/bin/bash
# r02ai: where the slowest alpha 0.7 / 0.9 sweep queries spend their time (latency mode)
mkdir -p gpurun_out
timeout 900 python tools/slow_queries.py 0.7 0.9 0.3 > gpurun_out/r02ai_slow_queries.txt 2>&1
