#!/bin/bash
# r02y: A/B of the r02t build (841c5f7), bcdcef1 (Grp / Q in shared memory) and HEAD in latency mode
mkdir -p gpurun_out
for b in abtest/r02t abtest/bcd .; do
  echo "== $b" >> gpurun_out/r02y_ab.txt
  timeout 600 python tools/ab_builds.py $b >> gpurun_out/r02y_ab.txt 2>&1
done
timeout 900 python tools/batch_sweep.py C4 8 > gpurun_out/r02y_c4_batch_split.txt 2>&1
timeout 2400 python tools/exp_sweeps.py > gpurun_out/r02y_exp_sweeps.txt 2>&1
