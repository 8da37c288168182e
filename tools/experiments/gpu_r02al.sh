#!/bin/bash
# r02al: status-word reset threshold n/16 (HEAD, abtest/head) vs n/64 (working tree): latency + batch
mkdir -p gpurun_out
for b in abtest/head . abtest/head .; do
  echo "== $b" >> gpurun_out/r02al_ab.txt
  timeout 600 python tools/ab_builds.py $b >> gpurun_out/r02al_ab.txt 2>&1
done
