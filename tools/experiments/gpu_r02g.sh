#!/bin/bash
# r02g: compute-sanitizer evidence for the lock-free engine (Thm. V.2 benign races are in global memory;
# racecheck covers the shared-memory arenas / tiles, synccheck the barriers, memcheck + initcheck bounds
# and uninitialised reads), C1 all queries + a C2 sample, single launches and batches
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  n2=3; [ $tool = racecheck ] && n2=1
  timeout 2400 $CS --tool $tool --print-limit 50 python tools/sanitize_run.py 100 $n2 > gpurun_out/r02g_cs_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/r02g_cs_$tool.log
done
for f in gpurun_out/r02g_cs_*.log; do tail -n 4 $f; done
