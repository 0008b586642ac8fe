set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "solve_host" > gpurun_out/pytest_batch.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_batch.log
timeout 900 python bench.py --no-cpu > gpurun_out/bench_batch.json 2> gpurun_out/bench_batch.err; echo "bench rc=$?"; tail -1 gpurun_out/bench_batch.json | cut -c1-300; tail -3 gpurun_out/bench_batch.err
