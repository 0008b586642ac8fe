timeout 900 python -m pytest tests/test_gpu_dist.py -q -x > gpurun_out/b21_pytest.log 2>&1; echo "pytest rc=$?"; tail -30 gpurun_out/b21_pytest.log | cut -c1-300
timeout 300 python tools/time_dist.py 1000000
DDA_DIST_SCALED=0 timeout 300 python tools/time_dist.py 1000000
