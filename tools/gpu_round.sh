#!/bin/bash
# one gpurun call: build, GPU tests, phase summaries (both node orders), bench (both node orders)
# usage: bash tools/gpu_round.sh [tests] [phases] [bench] [benchnorl]
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
for what in "$@"; do
  case $what in
    tests) timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log ;;
    phases) timeout 300 python tools/phase_summary.py --relabel 1 > gpurun_out/ph_rl.txt 2>&1
            timeout 300 python tools/phase_summary.py --relabel 0 > gpurun_out/ph_norl.txt 2>&1 ;;
    bench) timeout 500 python bench.py --no-cpu-baseline > gpurun_out/bench_rl.log 2>&1 ;;
    benchfull) timeout 600 python bench.py > gpurun_out/bench_full.log 2>&1 ;;
    benchnorl) KGS_RELABEL=0 timeout 500 python bench.py --no-cpu-baseline > gpurun_out/bench_norl.log 2>&1 ;;
  esac
done
