python -c "import __graft_entry__ as g; g.build()"
python tools/ab_flag.py dda__set_sp_prefetch 0,1,2,4 1000000 5 > gpurun_out/ab_pf.json 2>&1; cat gpurun_out/ab_pf.json
timeout 900 python -m pytest tests/test_gpu_dist.py -x -q > gpurun_out/pytest_dist4.log 2>&1; echo "pytest dist rc=$?"; tail -5 gpurun_out/pytest_dist4.log
python tools/time_dist.py 1000000 > gpurun_out/time_dist.json 2>&1; cat gpurun_out/time_dist.json
timeout 600 python bench.py --force-dist --steps 3 --warmup 3 --no-e2e > gpurun_out/bench_forcedist.json 2> gpurun_out/bench_forcedist.err; echo "bench force-dist rc=$?"; tail -2 gpurun_out/bench_forcedist.json; tail -3 gpurun_out/bench_forcedist.err
