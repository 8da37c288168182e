#!/bin/bash
# r02v: per-candidate cut-off validity (mk_reach), the cut inside a round / on overflow, deferred queries:
# parity, the C4 level-5 queries one by one, the C4 batch (deferral on / off), the C3 bench launch; then
# the L2 fetch-granularity experiment
mkdir -p gpurun_out
timeout 900 python -m pytest -x -q -p no:cacheprovider tests/test_gpu_prune.py tests/test_gpu_parity.py > gpurun_out/r02v_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02v_pytest.log
RECS=1,0 timeout 900 python tools/c4_one.py 2683 2906 11 1422 > gpurun_out/r02v_c4_one.txt 2>&1
timeout 900 python tools/batch_sweep.py C4 8,16 > gpurun_out/r02v_c4_batch.txt 2>&1
PARAMS="defer_min=0" timeout 900 python tools/batch_sweep.py C4 8 >> gpurun_out/r02v_c4_batch.txt 2>&1
timeout 900 python tools/batch_sweep.py C3 8,12 >> gpurun_out/r02v_c4_batch.txt 2>&1
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02v_pb8.log 2>&1
timeout 1500 python -m pytest -x -q -p no:cacheprovider "tests/test_gpu_fullsize.py::test_c4_sample_with_level5_queries" > gpurun_out/r02v_pytest_c4.log 2>&1; echo "rc=$?" >> gpurun_out/r02v_pytest_c4.log
bash tools/gpu_r02u.sh
