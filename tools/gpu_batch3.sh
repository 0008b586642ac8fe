NVAR=5 timeout 300 python tools/tune_spmv.py > gpurun_out/tune3.log 2>&1
for v in 0 1 2; do DDA_GSPMV_VARIANT=$v timeout 200 python tools/time_phases.py > gpurun_out/phases3_$v.log 2>&1; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/pytest_par3.log 2>&1
cat gpurun_out/tune3.log gpurun_out/phases3_*.log; tail -3 gpurun_out/pytest_par3.log
