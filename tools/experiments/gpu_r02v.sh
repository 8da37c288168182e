#!/bin/bash
# r02v: per-candidate cut-off validity (mk_reach), the cut inside a round / on overflow, deferred queries:
# parity, the C4 level-5 queries one by one, the C4 batch (deferral on / off), the C3 bench launch and its
# single-pass DRAM capture; then the L2 fetch-granularity experiment.  Usage: gpu_r02v.sh SHA
SHA=${1:-unknown}
mkdir -p gpurun_out/profiles
timeout 900 python -m pytest -x -q -p no:cacheprovider --durations=15 tests/test_gpu_prune.py tests/test_gpu_parity.py > gpurun_out/r02v_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02v_pytest.log
RECS=1,0 timeout 900 python tools/c4_one.py 2683 2906 11 1422 > gpurun_out/r02v_c4_one.txt 2>&1
timeout 900 python tools/batch_sweep.py C4 8,16 > gpurun_out/r02v_c4_batch.txt 2>&1
PARAMS="defer_min=0" timeout 900 python tools/batch_sweep.py C4 8 >> gpurun_out/r02v_c4_batch.txt 2>&1
timeout 900 python tools/batch_sweep.py C3 8,12 >> gpurun_out/r02v_c4_batch.txt 2>&1
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02v_pb8.log 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_engine -s 1 -c 1 --csv --log-file gpurun_out/r02v_traffic.csv python tools/profile_batch.py C3 350 8 > gpurun_out/r02v_traffic_pb.log 2>&1
python tools/make_traffic.py r02v gpurun_out/r02v_traffic.csv gpurun_out/r02v_traffic_pb.log 350 $SHA C3 > gpurun_out/r02v_make_traffic.log 2>&1
cp profiles/r02v_batch_traffic.json gpurun_out/profiles/ 2>/dev/null
timeout 1500 python -m pytest -x -q -p no:cacheprovider --durations=5 "tests/test_gpu_fullsize.py::test_c4_sample_with_level5_queries" > gpurun_out/r02v_pytest_c4.log 2>&1; echo "rc=$?" >> gpurun_out/r02v_pytest_c4.log
bash tools/experiments/gpu_r02u.sh
