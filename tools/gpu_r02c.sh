python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_dist.py tests/test_gpu_contacts.py -x -q > gpurun_out/pytest_c.log 2>&1; echo "pytest dist+contacts rc=$?"; tail -15 gpurun_out/pytest_c.log
mkdir -p gpurun_out/san2
run() {  # tool case tag envs...
  tool=$1; c=$2; tag=$3; shift 3
  env "$@" timeout 600 compute-sanitizer --tool $tool --print-limit 10 --error-exitcode 9 python tools/sanitize_cases.py tiny $c > gpurun_out/san2/${tool}_${c}_${tag}.log 2>&1
  echo "$tool $c $tag rc=$? $(grep -h SUMMARY gpurun_out/san2/${tool}_${c}_${tag}.log | tr '\n' ' ')"
}
run synccheck bj_graph base
run synccheck bj_graph pdl0 DDA_PDL=0
run synccheck bj_graph body1 DDA_BODY_ITERS=1
run synccheck bj_graph v4 DDA_GSPMV_VARIANT=1
run memcheck bj_graph base
run memcheck bj_graph pdl0 DDA_PDL=0
run memcheck bj_graph v4 DDA_GSPMV_VARIANT=1
run racecheck bj_scaled_graph pdl0 DDA_PDL=0
run initcheck bj_scaled_persistent base
run memcheck ilu0 pdl0 DDA_PDL=0
