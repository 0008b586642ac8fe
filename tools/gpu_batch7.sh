for v in 0 3; do DDA_GSPMV_VARIANT=$v timeout 200 python tools/time_phases.py 2>&1 | tail -1; done
for cfg in "DDA_GSPMV_VARIANT=0" "DDA_GSPMV_VARIANT=3" "DDA_GSPMV_VARIANT=1"; do
  env $cfg timeout 120 python tools/time_solve.py 1000000 5 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['env'], d['iters'], round(d['ms_median'],2), round(d['us_per_iter'],1))"
done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1
