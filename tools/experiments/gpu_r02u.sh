#!/bin/bash
# r02u: L2 fetch granularity (cudaLimitMaxL2FetchGranularity) on random gathers and on the bench launch
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/rgb tools/rand_gather_bench.cu
for g in 0 32 64 128; do
  echo "== gran $g" >> gpurun_out/r02u_rgb.txt
  /tmp/rgb $g >> gpurun_out/r02u_rgb.txt 2>&1
  timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r02u_rgb_ncu_$g.csv /tmp/rgb $g > /dev/null 2>&1
done
for g in 0 32 64 128; do
  L2GRAN=$g timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02u_pb_$g.log 2>&1
done
for g in 32 128; do
  L2GRAN=$g timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_engine --csv --log-file gpurun_out/r02u_pbncu_$g.csv python tools/profile_batch.py C3 350 8 > /dev/null 2>&1
done
