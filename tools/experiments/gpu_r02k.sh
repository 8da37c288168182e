#!/bin/bash
# r02k: where the top-down tail goes: the C4 level-5 queries one at a time (latency mode, phases), the NEXT-4
# sweeps with the paper's phase split and oracle parity at every point
mkdir -p gpurun_out
RECS=1 timeout 900 python tools/c4_one.py 2683 2906 11 1422 > gpurun_out/r02k_c4_one.txt 2>&1
timeout 1800 python tools/exp_sweeps.py 30 2 > gpurun_out/r02k_exp_sweeps.txt 2>&1
# A/B: the engine compiled for 3 CTAs per SM (40 registers, spills) against the default 2 (64 registers)
KGS_LIB=$PWD/build_ab/libkgs_minb3.so timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02k_pb_minb3.log 2>&1
KGS_LIB=$PWD/build_ab/libkgs_minb3.so timeout 600 python tools/profile_batch.py C3 350 12 > gpurun_out/r02k_pb_minb3_g12.log 2>&1
KGS_LIB=$PWD/build_ab/libkgs_minb3.so timeout 600 python tools/profile_batch.py C3 350 8 search_only=1 > gpurun_out/r02k_pb_minb3_so.log 2>&1
