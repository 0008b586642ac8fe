NVAR=6 timeout 300 python tools/tune_spmv.py > gpurun_out/tune4.log 2>&1
for v in 0 3 4; do DDA_GSPMV_VARIANT=$v timeout 200 python tools/time_phases.py > gpurun_out/phases4_$v.log 2>&1; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/pytest_par4.log 2>&1
cat gpurun_out/tune4.log; for v in 0 3 4; do echo "gspmv variant $v"; cat gpurun_out/phases4_$v.log; done; tail -3 gpurun_out/pytest_par4.log
