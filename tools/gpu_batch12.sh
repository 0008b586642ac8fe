timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/b12_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/b12_pytest.log
timeout 400 python tools/ab_loops.py 1000000 5
timeout 300 python tools/trace_loop.py 1000000 | cut -c1-600
timeout 300 python tools/time_phases.py 1000000 2>&1 | tail -2
