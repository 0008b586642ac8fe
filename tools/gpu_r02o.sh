python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_open_close.py tests/test_gpu_parity.py -q -k "transfer or ilu0 or precond_apply" > gpurun_out/pytest_o.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_o.log
for lib in ab_libs/libdda_head.so paper_conf_ipps_xiaohmxw17_b200/libdda.so; do
  DDA_LIB_PATH=$lib python tools/precond_study.py 100000 2>&1 | grep ilu0 | sed "s|^|$lib |"
done
