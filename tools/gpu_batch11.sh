timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/b11_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/b11_pytest.log
for cfg in "DDA_SCALED_LOOP=graph" "DDA_SCALED_LOOP=persist" "DDA_SCALED_LOOP=graph" "DDA_SCALED_LOOP=persist"; do
  env $cfg timeout 120 python tools/time_solve.py 1000000 5 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg', d['iters'], d['rel'], round(d['ms_median'],2), round(d['us_per_iter'],1))"
done
timeout 300 python tools/trace_loop.py 1000000
python - <<'PY'
import sys; sys.path.insert(0,'.')
import torch, paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
P = make_slope(preset(1000000, seed=1005)); t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"]); K.bj_setup()
d, it, rr, st = K.pcg_solve(t["F"]); print("checks", K.last_checks(), "iters", it)
PY
