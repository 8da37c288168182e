#!/bin/bash
# r02c: the GPU suite (fullsize last), smoke, the overlap probe for NEXT-1, ncu timing of the batch launch
# with and without ncu's cache control (the 86 ms vs 116 ms question)
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --deselect tests/test_gpu_fullsize.py > gpurun_out/r02c_pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02c_pytest_gpu.log
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider > gpurun_out/r02c_pytest_full.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02c_pytest_full.log
timeout 900 python tools/overlap_probe.py 8 4 > gpurun_out/r02c_overlap.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:k_engine --csv --log-file gpurun_out/r02c_ncu_nocache.csv python tools/profile_batch.py C3 350 8 > gpurun_out/r02c_pb1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control all -k regex:k_engine --csv --log-file gpurun_out/r02c_ncu_cacheall.csv python tools/profile_batch.py C3 350 8 > gpurun_out/r02c_pb2.log 2>&1
tail -3 gpurun_out/r02c_pytest_gpu.log gpurun_out/r02c_pytest_full.log gpurun_out/r02c_overlap.txt
