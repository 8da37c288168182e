#!/bin/bash
# r02h: fire-and-forget hits (no returned atomic in visit_arc): GPU suite + batch timing, then the sanitizers
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider --deselect tests/test_gpu_fullsize.py > gpurun_out/r02h_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02h_pytest.log
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02h_pb.log 2>&1
timeout 600 python tools/profile_batch.py C3 350 8 search_only=1 > gpurun_out/r02h_pb_so.log 2>&1
for G in 4 6 12; do timeout 600 python tools/profile_batch.py C3 350 $G > gpurun_out/r02h_pb_g$G.log 2>&1; done
bash tools/experiments/gpu_r02g.sh
