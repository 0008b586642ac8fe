nvidia-smi --query-gpu=name,driver_version,clocks.max.sm --format=csv > gpurun_out/clean_build.log
( time python -c "from paper_conf_ipps_xiaohmxw17_b200 import _build; _build.build(force=True, verbose=True)" ) >> gpurun_out/clean_build.log 2>&1; echo "clean build rc=$?"
cuobjdump -lelf paper_conf_ipps_xiaohmxw17_b200/libdda.so 2>&1 | head -5 >> gpurun_out/clean_build.log
cuobjdump -sass paper_conf_ipps_xiaohmxw17_b200/libdda.so | grep -c 'LDG.E.NA.ENL2.256' >> gpurun_out/clean_build.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
mkdir -p gpurun_out/san4
for tool in memcheck racecheck synccheck initcheck; do
  timeout 600 compute-sanitizer --tool $tool --print-limit 10 --error-exitcode 9 python tools/sanitize_cases.py tiny dist > gpurun_out/san4/${tool}_tiny_dist.log 2>&1
  echo "$tool tiny dist(v4) rc=$? $(grep -h SUMMARY gpurun_out/san4/${tool}_tiny_dist.log | tr '\n' ' ')"
done
DDA_TRACE=1 timeout 600 python tools/open_close.py 1000000 3 > gpurun_out/open_close.json 2> gpurun_out/open_close_trace.log; echo "open_close rc=$?"; cat gpurun_out/open_close.json | cut -c1-1500
