python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests/test_gpu_dist.py -x -q > gpurun_out/pytest_dist6.log 2>&1; echo "pytest dist rc=$?"; tail -3 gpurun_out/pytest_dist6.log
python tools/time_dist.py 1000000 > gpurun_out/time_dist.json 2>&1; cat gpurun_out/time_dist.json
timeout 600 compute-sanitizer --tool racecheck --print-limit 10 --error-exitcode 9 env DDA_DIST_VERSION=4 python tools/sanitize_cases.py tiny dist > gpurun_out/san_dist_ovl.log 2>&1; echo "racecheck v4 overlap rc=$? $(grep -h SUMMARY gpurun_out/san_dist_ovl.log)"
timeout 600 compute-sanitizer --tool memcheck --print-limit 10 --error-exitcode 9 env DDA_DIST_VERSION=4 python tools/sanitize_cases.py tiny dist > gpurun_out/san_dist_ovl2.log 2>&1; echo "memcheck v4 overlap rc=$? $(grep -h SUMMARY gpurun_out/san_dist_ovl2.log)"
