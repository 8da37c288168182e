#!/bin/bash
# NEXT-2 after the 128-pair / one-sector change: parity, C3 timing, launch list with DRAM bytes
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_prep.py -x -q > gpurun_out/pytest_prep.log 2>&1; echo rc=$? >> gpurun_out/pytest_prep.log
timeout 600 python tools/prep_bench.py > gpurun_out/prep_bench.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_dist|k_summary|k_normalise|DeviceSegmented" --csv --log-file gpurun_out/prep_launches.csv python tools/prep_bench.py 128 > gpurun_out/prep_ncu.log 2>&1
echo done
