python -c "import __graft_entry__ as g; g.build()"
for lib in ab_libs/libdda_head.so paper_conf_ipps_xiaohmxw17_b200/libdda.so ab_libs/libdda_head.so paper_conf_ipps_xiaohmxw17_b200/libdda.so; do
  DDA_LIB_PATH=$lib python tools/time_build.py 1000000 | sed "s|^|$lib |"
done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -k "assembly or update_values or golden or no_springs or invalid or fullsize_assembly" > gpurun_out/pytest_asm.log 2>&1; echo "pytest asm rc=$?"; tail -3 gpurun_out/pytest_asm.log
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --csv -k regex:"k_pack|k_offdiag|k_diag|k_rank|k_dkeys" python tools/time_build.py 1000000 > gpurun_out/asm_ncu.csv 2>&1; echo "ncu rc=$?"; grep -E 'k_pack|k_offdiag_r|k_diag_r' gpurun_out/asm_ncu.csv | head -12
