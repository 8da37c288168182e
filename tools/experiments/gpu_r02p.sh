#!/bin/bash
mkdir -p gpurun_out
for G in 8 12 16; do timeout 600 python tools/profile_batch.py C3 350 $G > gpurun_out/r02p_pb$G.log 2>&1; done
timeout 900 python tools/phase_summary.py --config C3 --queries 120 > gpurun_out/r02p_phases.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider --deselect tests/test_gpu_fullsize.py --deselect tests/test_gpu_sweeps.py::test_c3_sweep_points > gpurun_out/r02p_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02p_pytest.log
