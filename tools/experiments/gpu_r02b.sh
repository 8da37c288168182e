#!/bin/bash
# r02b: the whole GPU suite + smoke after the parity round (R15 oracle snap, R6, new full-size tests)
mkdir -p gpurun_out
timeout 3000 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/r02b_pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02b_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02b_smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/r02b_smoke.log
timeout 600 python tools/workload_scan.py C4 > gpurun_out/r02b_c4_scan.txt 2>&1
tail -5 gpurun_out/r02b_pytest_gpu.log gpurun_out/r02b_smoke.log
