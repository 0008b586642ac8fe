set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 1200 python -m pytest tests/test_gpu_dist.py -m gpu -x -q > gpurun_out/pytest_dist_v6.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_dist_v6.log
timeout 900 python tools/time_dist.py 1000000 > gpurun_out/time_dist_v6.json 2>&1; tail -c 300 gpurun_out/time_dist_v6.json
rm -rf gpurun_out/san; SAN_SIZES=tiny SAN_CASES="dist" bash tools/gpu_sanitize.sh
