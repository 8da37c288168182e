make -j8 all >/dev/null 2>&1
for rl in 1 0; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_engine -s 7 -c 1 -o gpurun_out/heavy_rl$rl python tools/profile_run.py --warm 7 --queries 1 --relabel $rl > gpurun_out/ncu_heavy_rl$rl.log 2>&1
done
