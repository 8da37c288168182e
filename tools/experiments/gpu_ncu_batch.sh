#!/bin/bash
# one --set full capture of a batch-mode engine launch (the bench's launch shape, 350 queries, G=8) and of
# one latency-mode query (bench order query 41, G=1)
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_engine -s 1 -c 1 -o gpurun_out/batch_full -f python tools/profile_batch.py C3 350 8 > gpurun_out/ncu_batch.log 2>&1
ncu -i gpurun_out/batch_full.ncu-rep --page details --csv > gpurun_out/batch_details.csv 2>&1
ncu -i gpurun_out/batch_full.ncu-rep --page raw --csv > gpurun_out/batch_raw.csv 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_engine -s 41 -c 1 -o gpurun_out/lat_full -f python tools/profile_run.py --warm 41 --queries 1 > gpurun_out/ncu_lat.log 2>&1
