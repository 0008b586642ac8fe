# persistent scaled loop vs graph loop: parity + timing
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/b10_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/b10_pytest.log
for cfg in "DDA_SCALED_LOOP=graph" "DDA_SCALED_LOOP=persist" "DDA_SCALED_LOOP=graph" "DDA_SCALED_LOOP=persist"; do
  env $cfg timeout 120 python tools/time_solve.py 1000000 5 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg', d['iters'], d['rel'], round(d['ms_median'],2), round(d['us_per_iter'],1))"
done
timeout 600 python bench.py --no-cpu > gpurun_out/b10_bench.json 2> gpurun_out/b10_bench.err; echo "bench rc=$?"; cat gpurun_out/b10_bench.json | head -c 1500
