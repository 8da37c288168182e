#!/bin/bash
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 600 python tools/pull_compare.py C5 6 > gpurun_out/pull_c5.txt 2>&1
timeout 600 python tools/pull_compare.py C3 30 > gpurun_out/pull_c3.txt 2>&1
KGS_LIB=paper_conf_icde_yangajtw19_b200/libkgs.so timeout 600 python tools/ab_perf.py > gpurun_out/ab.txt 2>&1
