#!/bin/bash
# r02j: records reverted; deferred-pass unroll; race / init fixes
mkdir -p gpurun_out
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02j_pb.log 2>&1
timeout 600 python tools/profile_batch.py C3 350 8 search_only=1 > gpurun_out/r02j_pb_so.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider --deselect tests/test_gpu_fullsize.py --deselect tests/test_gpu_sweeps.py::test_c3_sweep_points > gpurun_out/r02j_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02j_pytest.log
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool racecheck --print-limit 50 python tools/sanitize_run.py 100 1 > gpurun_out/r02j_cs_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02j_cs_racecheck.log
timeout 1200 $CS --tool initcheck --print-limit 50 python tools/sanitize_run.py 30 0 > gpurun_out/r02j_cs_initcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02j_cs_initcheck.log
