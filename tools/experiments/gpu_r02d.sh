#!/bin/bash
# r02d: random-access ceilings of this B200 (rand_gather_bench), search-only vs full batch DRAM bytes and
# time (the bench's launch shape), recorded DAG in batch mode, and the tests that failed in r02c
mkdir -p gpurun_out
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/rgb tools/rand_gather_bench.cu && /tmp/rgb > gpurun_out/r02d_rgb.txt 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --csv --log-file gpurun_out/r02d_rgb_ncu.csv /tmp/rgb > /dev/null 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct
for cfg in "full" "search_only=1" "dag_record=1"; do
  tag=$(echo $cfg | tr '=' '_')
  timeout 900 ncu --metrics $M --clock-control none -k regex:k_engine --csv --log-file gpurun_out/r02d_pb_$tag.csv python tools/profile_batch.py C3 350 8 $( [ "$cfg" != full ] && echo $cfg ) > gpurun_out/r02d_pb_$tag.log 2>&1
done
timeout 1800 python -m pytest -q -p no:cacheprovider tests/test_gpu_offgrid.py tests/test_gpu_prep.py tests/test_gpu_next3.py "tests/test_gpu_fullsize.py::test_tier4_extraction" tests/test_gpu_parity.py > gpurun_out/r02d_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02d_pytest.log
