python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_dist.py -x -q > gpurun_out/pytest_dist5.log 2>&1; echo "pytest dist rc=$?"; tail -3 gpurun_out/pytest_dist5.log
python tools/time_dist.py 1000000 > gpurun_out/time_dist.json 2>&1; cat gpurun_out/time_dist.json
for tool in memcheck racecheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool --print-limit 10 --error-exitcode 9 python tools/sanitize_cases.py tiny dist > gpurun_out/san_dist5_$tool.log 2>&1
  echo "$tool tiny dist(v5) rc=$? $(grep -h SUMMARY gpurun_out/san_dist5_$tool.log | tr '\n' ' ')"
done
