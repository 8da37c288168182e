#!/bin/bash
# r02l: latency-mode phase split by query class (where small queries' fixed cost goes) + one ncu --set full
# capture of the bench's batch launch on the current build (hot lines)
mkdir -p gpurun_out
timeout 900 python tools/phase_summary.py --config C3 --queries 120 > gpurun_out/r02l_phases.txt 2>&1
timeout 1800 ncu --set full --import-source on --clock-control none -k regex:k_engine -s 1 -c 1 -o gpurun_out/r02l_batch -f python tools/profile_batch.py C3 350 8 > gpurun_out/r02l_ncu.log 2>&1
python tools/ncu_hot.py gpurun_out/r02l_batch.ncu-rep k_engine 60 > gpurun_out/r02l_hot.txt 2>&1
ncu -i gpurun_out/r02l_batch.ncu-rep --page details --csv > gpurun_out/r02l_details.csv 2>&1
ncu -i gpurun_out/r02l_batch.ncu-rep --page raw --csv > gpurun_out/r02l_raw.csv 2>&1
rm -f gpurun_out/r02l_batch.ncu-rep
