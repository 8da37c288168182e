timeout 900 python -m pytest -q -p no:cacheprovider tests/test_gpu_parity.py -k "across_launches" > gpurun_out/r02e_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02e_pytest.log
timeout 600 python tools/profile_batch.py C3 350 8 dag_record=1 > gpurun_out/r02e_pb_rec.log 2>&1
timeout 600 python tools/profile_batch.py C3 350 8 search_only=1 > gpurun_out/r02e_pb_so.log 2>&1
for pm in 64 160 512; do timeout 600 python tools/profile_batch.py C3 350 8 prune_min=$pm > gpurun_out/r02e_pb_pm$pm.log 2>&1; done
