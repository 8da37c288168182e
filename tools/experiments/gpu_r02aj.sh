#!/bin/bash
# r02aj: a large recorded DAG is dropped for the pre-pass + lazy round 2 when pruning runs (rec_max):
# parity, the slow sweep queries, the sweeps, latency p50 (bench latency mode) and the C4 batch
mkdir -p gpurun_out
timeout 900 python -m pytest -x -q -p no:cacheprovider tests/test_gpu_prune.py tests/test_gpu_parity.py tests/test_gpu_direction.py tests/test_gpu_next3.py > gpurun_out/r02aj_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02aj_pytest.log
timeout 900 python tools/slow_queries.py 0.9 > gpurun_out/r02aj_slow_queries.txt 2>&1
timeout 1800 python tools/exp_sweeps.py > gpurun_out/r02aj_exp_sweeps.txt 2>&1
timeout 900 python tools/batch_sweep.py C4 8 > gpurun_out/r02aj_c4.txt 2>&1
