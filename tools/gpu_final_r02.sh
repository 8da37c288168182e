#!/bin/bash
# The round's evidence run: GPU suite, smoke, bench line (C4: 4096 queries per step), the bench's ncu launch
# list, a single-pass DRAM capture of the bench-shaped launch (roofline.traffic) and one ncu --set full
# capture of it (sections + per-line stalls) -> profiles/<tag>_*.  Usage: gpu_final_r02.sh SHA [TAG]
SHA=${1:-unknown}
TAG=${2:-r02}
W=C4; NQ=4096
mkdir -p gpurun_out/profiles
timeout 3000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout=1200 --durations=30 > gpurun_out/fin_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/fin_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fin_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/fin_smoke.log
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fin_launches.csv python bench.py --steps 2 --warmup 3 --latency-steps 20 --no-cpu-baseline > gpurun_out/fin_ncu_bench.log 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_engine -s 1 -c 1 --csv --log-file gpurun_out/fin_traffic.csv python tools/profile_batch.py $W $NQ 8 > gpurun_out/fin_traffic_pb.log 2>&1
python tools/make_traffic.py $TAG gpurun_out/fin_traffic.csv gpurun_out/fin_traffic_pb.log $NQ $SHA $W > gpurun_out/fin_make_traffic.log 2>&1
timeout 1200 python bench.py > gpurun_out/fin_bench.json 2> gpurun_out/fin_bench.err
timeout 1200 python bench.py --workload C3 --no-cpu-baseline > gpurun_out/fin_bench_c3.json 2> gpurun_out/fin_bench_c3.err
timeout 1800 ncu --set full --import-source on --clock-control none -k regex:k_engine -s 1 -c 1 -o gpurun_out/fin_batch -f python tools/profile_batch.py C3 350 8 > gpurun_out/fin_ncu_batch.log 2>&1
ncu -i gpurun_out/fin_batch.ncu-rep --page details --csv > gpurun_out/fin_batch_details.csv 2>&1
ncu -i gpurun_out/fin_batch.ncu-rep --page raw --csv > gpurun_out/fin_batch_raw.csv 2>&1
python tools/ncu_hot.py gpurun_out/fin_batch.ncu-rep k_engine 45 > gpurun_out/fin_batch_hot.txt 2>&1
python tools/make_batch_profile.py $TAG gpurun_out/fin_batch_details.csv gpurun_out/fin_batch_raw.csv gpurun_out/fin_batch_hot.txt 350 $SHA C3 > gpurun_out/fin_mbp.log 2>&1
cp profiles/${TAG}_batch_* gpurun_out/profiles/ 2>/dev/null
tail -3 gpurun_out/fin_pytest.log gpurun_out/fin_smoke.log; cat gpurun_out/fin_bench.json
timeout 1800 python tools/exp_sweeps.py > gpurun_out/fin_exp_sweeps.txt 2>&1
