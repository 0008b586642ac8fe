timeout 900 python -m pytest tests/test_gpu_contacts.py -q -x > gpurun_out/b18_pytest.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/b18_pytest.log
timeout 300 python tools/time_contacts.py 1000000 0.2 | tee gpurun_out/contacts_1m.json
timeout 300 python tools/time_contacts.py 10000 0.2
