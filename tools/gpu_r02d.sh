python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests/test_gpu_dist.py tests/test_gpu_contacts.py tests/test_gpu_open_close.py -q > gpurun_out/pytest_d.log 2>&1; echo "pytest rc=$?"; tail -25 gpurun_out/pytest_d.log
mkdir -p gpurun_out/san3
for tool in memcheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool --print-limit 10 --error-exitcode 9 python tools/sanitize_cases.py tiny bj_graph_phases > gpurun_out/san3/${tool}_phases.log 2>&1
  echo "$tool phases rc=$? $(grep -h SUMMARY gpurun_out/san3/${tool}_phases.log | tr '\n' ' ')"
  grep -v 'Host Frame' gpurun_out/san3/${tool}_phases.log | head -12
done
