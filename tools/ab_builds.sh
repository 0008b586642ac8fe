# Two-build A/B of libdda.so on one GPU box (k_sp_loop runs at its 80-register cap, so
# in-kernel runtime switches perturb its code generation; compare separate builds instead).
# usage: bash tools/ab_builds.sh "<nvcc flags A>" "<nvcc flags B>" [rounds] [n]
#   e.g. bash tools/ab_builds.sh "" "-DDDA_TR_EVICT_FIRST" 2
# Per build and round: the BJ solve (tools/time_solve.py), its per-phase timeline (tools/trace_loop.py) and
# the standalone SpMV (tools/spmv_ab.py); the default build is restored at the end.
A="$1"; Bf="$2"; R="${3:-2}"; N="${4:-1000000}"
BUILD=paper_conf_ipps_xiaohmxw17_b200/_build.py
run() {
  timeout 300 python tools/time_solve.py "$N" 6 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('$1 solve', d['iters'], round(d['us_per_iter'],1), round(d['ms_median'],2))"
  timeout 300 python tools/trace_loop.py "$N" | python -c "import json,sys;d=json.loads(sys.stdin.read());print('$1 trace', {k: d[k] for k in ('iter_us','phaseA_cta_median_us','phaseA_end_spread_us','barrier1_median_wait_us','phaseB_cta_median_us','barrier2_median_wait_us')})"
  timeout 300 python tools/spmv_ab.py "X=0" "$N" 20 2>&1 | python -c "import json,sys;d=json.loads(sys.stdin.read().strip().splitlines()[-1]);r=d['results'][0];print('$1 spmv', round(r['ms']*1000,1), round(r['frac'],3))"
}
for r in $(seq "$R"); do
  python $BUILD $A > /dev/null 2>&1; run A
  python $BUILD $Bf > /dev/null 2>&1; run B
done
python $BUILD > /dev/null 2>&1
