timeout 900 python -m pytest tests/test_gpu_dist.py -x -q > gpurun_out/pytest_dist.log 2>&1; echo "pytest dist rc=$?"; tail -15 gpurun_out/pytest_dist.log
SAN_SIZES=tiny bash tools/gpu_sanitize.sh
