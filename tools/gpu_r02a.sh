timeout 1500 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -x -q -k "z17 or update_values or bj_inverse" > gpurun_out/pytest_r02a.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_r02a.log
bash tools/gpu_sanitize.sh
