#!/bin/bash
# A/B of prebuilt libkgs variants in build_var/ (built on the CPU side)
mkdir -p gpurun_out
for v in ${VARIANTS:-D A B C}; do
  KGS_LIB=build_var/libkgs_$v.so timeout 600 python tools/ab_perf.py >> gpurun_out/ab.txt 2>&1
done
