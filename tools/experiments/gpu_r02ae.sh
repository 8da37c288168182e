#!/bin/bash
# r02ae: reproduce the r02ad two-rank crash in one process, isolate lazy DAG / deferral; q = 8 lazy parity
mkdir -p gpurun_out
for v in default nolazy nodefer both; do
  timeout 600 python tools/repro_2rank.py $v 4 >> gpurun_out/r02ae_repro.txt 2>&1; echo "$v rc=$?" >> gpurun_out/r02ae_repro.txt
done
timeout 900 python -m pytest -x -q -p no:cacheprovider tests/test_gpu_prune.py tests/test_gpu_parity.py > gpurun_out/r02ae_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02ae_pytest.log
