for cfg in "DDA_GSPMV_VARIANT=0" "DDA_GSPMV_VARIANT=4" "DDA_GSPMV_VARIANT=5" "DDA_GSPMV_VARIANT=3" "DDA_GSPMV_VARIANT=0"; do
  env $cfg timeout 120 python tools/time_solve.py 1000000 5 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['env'], d['iters'], d['rel'], round(d['ms_median'],2), round(d['us_per_iter'],1))"
done
