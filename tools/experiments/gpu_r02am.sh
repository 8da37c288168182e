#!/bin/bash
# r02am: ncu --set full of the C4 bench launch (4096 queries, G = 8): sections + per-line stalls
SHA=${1:-unknown}
mkdir -p gpurun_out/profiles
timeout 2400 ncu --set full --import-source on --clock-control none -k regex:k_engine -s 1 -c 1 -o gpurun_out/c4_batch -f python tools/profile_batch.py C4 4096 8 > gpurun_out/c4_ncu_batch.log 2>&1
ncu -i gpurun_out/c4_batch.ncu-rep --page details --csv > gpurun_out/c4_batch_details.csv 2>&1
ncu -i gpurun_out/c4_batch.ncu-rep --page raw --csv > gpurun_out/c4_batch_raw.csv 2>&1
python tools/ncu_hot.py gpurun_out/c4_batch.ncu-rep k_engine 45 > gpurun_out/c4_batch_hot.txt 2>&1
python tools/make_batch_profile.py r02c4 gpurun_out/c4_batch_details.csv gpurun_out/c4_batch_raw.csv gpurun_out/c4_batch_hot.txt 4096 $SHA C4 > gpurun_out/c4_mbp.log 2>&1
cp profiles/r02c4_batch_* gpurun_out/profiles/ 2>/dev/null
grep launch gpurun_out/c4_ncu_batch.log >> gpurun_out/profiles/r02c4_batch_ncu.md
