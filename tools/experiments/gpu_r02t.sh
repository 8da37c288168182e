#!/bin/bash
mkdir -p gpurun_out
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02t_pb8.log 2>&1
timeout 900 python tools/batch_sweep.py C3 8,12 > gpurun_out/r02t_sweep.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider --deselect tests/test_gpu_fullsize.py --deselect tests/test_gpu_sweeps.py::test_c3_sweep_points > gpurun_out/r02t_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02t_pytest.log
