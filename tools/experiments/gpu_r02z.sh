#!/bin/bash
# r02z: where the pruning rounds spend the C4 batch (round-2 phase stamps)
mkdir -p gpurun_out
timeout 900 python tools/batch_sweep.py C4 8 > gpurun_out/r02z_c4_split.txt 2>&1
PARAMS="prune_min=4096" timeout 900 python tools/batch_sweep.py C4 8 >> gpurun_out/r02z_c4_split.txt 2>&1
