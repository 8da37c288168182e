make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 600 python tools/profile_run.py --config C5 --warm 0 --queries 10 > gpurun_out/c5_phases.log 2>&1
KGS_DAG_RECORD=0 timeout 600 python tools/profile_run.py --config C5 --warm 0 --queries 10 > gpurun_out/c5_phases_norec.log 2>&1
