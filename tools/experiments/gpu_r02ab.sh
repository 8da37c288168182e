#!/bin/bash
# r02ab: lazy round-2 DAG (kgs_params.lazy_dag): parity, then C4 / C3 batches with lazy on / off
mkdir -p gpurun_out
timeout 900 python -m pytest -x -q -p no:cacheprovider --durations=10 tests/test_gpu_prune.py tests/test_gpu_parity.py tests/test_gpu_next3.py tests/test_gpu_direction.py tests/test_gpu_offgrid.py > gpurun_out/r02ab_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02ab_pytest.log
timeout 900 python tools/batch_sweep.py C4 8 > gpurun_out/r02ab_split.txt 2>&1
PARAMS="lazy_dag=0" timeout 900 python tools/batch_sweep.py C4 8 >> gpurun_out/r02ab_split.txt 2>&1
timeout 900 python tools/batch_sweep.py C3 8 >> gpurun_out/r02ab_split.txt 2>&1
PARAMS="lazy_dag=0" timeout 900 python tools/batch_sweep.py C3 8 >> gpurun_out/r02ab_split.txt 2>&1
RECS=1,0 timeout 900 python tools/c4_one.py 2683 2906 11 > gpurun_out/r02ab_c4_one.txt 2>&1
timeout 1500 python -m pytest -x -q -p no:cacheprovider tests/test_gpu_fullsize.py tests/test_gpu_sweeps.py > gpurun_out/r02ab_pytest_full.log 2>&1; echo "rc=$?" >> gpurun_out/r02ab_pytest_full.log
