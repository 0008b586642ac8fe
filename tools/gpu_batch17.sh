timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/b17_pytest.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/b17_pytest.log
timeout 500 python tools/ab_loops.py 1000000 4 | cut -c1-700
timeout 300 python tools/trace_loop.py 1000000 2 | cut -c1-700
