#!/bin/bash
# r02aa: rm bits in the status word (the key cut-off's validity from the search), fix of the mk_reach
# lookup; parity (incl. the hand-built s* = 2 winner), C4 sample, batch sweeps, level-5 queries
mkdir -p gpurun_out
timeout 900 python -m pytest -x -q -p no:cacheprovider --durations=10 tests/test_gpu_prune.py tests/test_gpu_parity.py tests/test_gpu_next3.py tests/test_gpu_direction.py > gpurun_out/r02aa_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02aa_pytest.log
timeout 900 python tools/batch_sweep.py C4 8 > gpurun_out/r02aa_c4_split.txt 2>&1
timeout 900 python tools/batch_sweep.py C3 8 >> gpurun_out/r02aa_c4_split.txt 2>&1
RECS=1 timeout 900 python tools/c4_one.py 2683 2906 11 > gpurun_out/r02aa_c4_one.txt 2>&1
timeout 1500 python -m pytest -x -q -p no:cacheprovider tests/test_gpu_fullsize.py > gpurun_out/r02aa_pytest_full.log 2>&1; echo "rc=$?" >> gpurun_out/r02aa_pytest_full.log
