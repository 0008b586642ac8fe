for n in 10000 30000; do
for cfg in "DDA_PCG_ENGINE=persistent" "DDA_PCG_ENGINE=scaled" "DDA_PCG_ENGINE=scaled DDA_PERSIST_CTAS=64" "DDA_PCG_ENGINE=scaled DDA_PERSIST_CTAS=32" "DDA_PCG_ENGINE=scaled DDA_PERSIST_CTAS=444"; do
  env $cfg timeout 120 python tools/time_solve.py $n 10 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print($n, '$cfg', d['iters'], round(d['ms_median'],3), round(d['us_per_iter'],2))"
done; done
