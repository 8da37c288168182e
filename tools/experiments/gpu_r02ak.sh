#!/bin/bash
# r02ak: where a latency-mode query's time goes at the end of the round (C4 and C3 bench order)
mkdir -p gpurun_out
timeout 900 python tools/phase_summary.py --config C3 --queries 200 > gpurun_out/r02ak_phases_c3.txt 2>&1
