for cfg in "DDA_BODY_ITERS=2" "DDA_BODY_ITERS=1" "DDA_BODY_ITERS=4" "DDA_BODY_ITERS=8" "DDA_PDL=0" "DDA_GSPMV_VARIANT=1" "DDA_BODY_ITERS=2"; do
  env $cfg timeout 120 python tools/time_solve.py 1000000 5 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['env'], d['iters'], round(d['ms_median'],2), round(d['us_per_iter'],1))"
done
