#!/bin/bash
# r02f: the st32 status word (hm | gate | nm | a in one word): GPU suite (not the full-size file), batch timing
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider --deselect tests/test_gpu_fullsize.py > gpurun_out/r02f_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02f_pytest.log
timeout 600 python tools/profile_batch.py C3 350 8 > gpurun_out/r02f_pb.log 2>&1
timeout 600 python tools/profile_batch.py C3 350 8 search_only=1 > gpurun_out/r02f_pb_so.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct
timeout 900 ncu --metrics $M --clock-control none -k regex:k_engine -s 1 -c 1 --csv --log-file gpurun_out/r02f_ncu.csv python tools/profile_batch.py C3 350 8 > /dev/null 2>&1
tail -2 gpurun_out/r02f_pytest.log; cat gpurun_out/r02f_pb.log gpurun_out/r02f_pb_so.log
