set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu3.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu3.log
timeout 400 python bench.py > gpurun_out/bench_s4.json 2> gpurun_out/bench_s4.err
timeout 600 ncu --graph-profiling graph --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --csv --log-file gpurun_out/graph_traffic_s.csv python tools/prof_case.py --spmv 1 --pcg-maxit 10000 > gpurun_out/prof_case1.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches_s.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --spmv-reps 3 > gpurun_out/bench_ncu.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_g_spmv --launch-skip 10 --launch-count 1 -o gpurun_out/spmv_sc python tools/prof_case.py --pcg-maxit 30 > gpurun_out/prof_spmv.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_s_update --launch-skip 10 --launch-count 1 -o gpurun_out/upd_sc python tools/prof_case.py --pcg-maxit 30 > gpurun_out/prof_upd.log 2>&1
ls -la gpurun_out
