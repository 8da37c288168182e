#!/bin/bash
# round-end evidence: GPU tests, full bench, bench launch list under ncu, one --set full capture of the
# bench-shaped batch launch (C4, 4096 queries, G=8)
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
if [ -z "$NO_TESTS" ]; then
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
fi
timeout 900 python bench.py > gpurun_out/bench_full.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_ --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --latency-steps 20 > gpurun_out/bench_ncu.log 2>&1
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:k_engine -s 1 -c 1 -o gpurun_out/batch_full -f python tools/profile_batch.py C3 350 8 > gpurun_out/ncu_batch.log 2>&1
ncu -i gpurun_out/batch_full.ncu-rep --page details --csv > gpurun_out/batch_details.csv 2>&1
ncu -i gpurun_out/batch_full.ncu-rep --page raw --csv > gpurun_out/batch_raw.csv 2>&1
echo done
