#!/bin/bash
# round-end check of the restored tree + the NEXT-2 preprocessing kernels: prep parity first, then the
# whole GPU suite, the bench, and the bench launch list under ncu.
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 600 python -m pytest tests/test_gpu_prep.py -x -q > gpurun_out/pytest_prep.log 2>&1; echo rc=$? >> gpurun_out/pytest_prep.log
timeout 300 python tools/prep_bench.py > gpurun_out/prep_bench.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_full.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_ --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --latency-steps 20 > gpurun_out/bench_ncu.log 2>&1
echo done
