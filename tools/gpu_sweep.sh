make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 600 python tools/batch_sweep.py C3 8,16,24,37,74 1400 > gpurun_out/sweep_auto.txt 2>&1
KGS_DAG_RECORD=1 timeout 600 python tools/batch_sweep.py C3 8,16,37,74 1400 > gpurun_out/sweep_rec.txt 2>&1
