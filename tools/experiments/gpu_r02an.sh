#!/bin/bash
# r02an: Python-side result export (lazy statistics, one list conversion per array): GPU suite + bench (e2e)
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout=1200 > gpurun_out/r02an_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02an_pytest.log
timeout 1200 python bench.py > gpurun_out/r02an_bench.json 2> gpurun_out/r02an_bench.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02an_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r02an_smoke.log
