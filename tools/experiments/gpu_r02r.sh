#!/bin/bash
mkdir -p gpurun_out
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02r_pb8.log 2>&1
timeout 900 python tools/phase_summary.py --config C3 --queries 120 > gpurun_out/r02r_phases.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider --deselect tests/test_gpu_fullsize.py --deselect tests/test_gpu_sweeps.py::test_c3_sweep_points > gpurun_out/r02r_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02r_pytest.log
