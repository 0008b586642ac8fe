timeout 900 python -m pytest tests/test_gpu_dist.py -q -x > gpurun_out/b19_pytest.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/b19_pytest.log
timeout 300 python tools/time_dist.py 1000000
DDA_DIST_CHUNK=1 timeout 300 python tools/time_dist.py 1000000
