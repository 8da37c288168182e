#!/bin/bash
# A/B of engine environment knobs with the in-tree build: ENVS="K=V;K=V ..." (space separates runs)
make -j8 all >/dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
for e in $ENVS; do
  echo "== $e" >> gpurun_out/env_ab.txt
  env $(echo $e | tr ';' ' ') timeout 600 python tools/ab_perf.py ${AB_ARGS:-150 1400 8} >> gpurun_out/env_ab.txt 2>&1
done
