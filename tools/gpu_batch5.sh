set -x
timeout 400 python bench.py > gpurun_out/bench_s8.json 2> gpurun_out/bench_s8.err
timeout 600 ncu --graph-profiling graph --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --csv --log-file gpurun_out/graph_traffic_s2.csv python tools/prof_case.py --spmv 1 --pcg-maxit 10000 > gpurun_out/prof_case2.log 2>&1
timeout 900 ncu --graph-profiling graph --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_s2.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --spmv-reps 3 > gpurun_out/bench_ncu2.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_g_spmv --launch-skip 2 --launch-count 1 -o gpurun_out/spmv_sc2 python tools/prof_phases.py 1000000 1 > gpurun_out/prof_spmv2.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_s_update --launch-skip 2 --launch-count 1 -o gpurun_out/upd_sc2 python tools/prof_phases.py 1000000 1 > gpurun_out/prof_upd2.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_spmv3 --launch-skip 3 --launch-count 1 -o gpurun_out/spmv_std2 python tools/prof_case.py --spmv 5 --pcg-maxit 1 > gpurun_out/prof_std2.log 2>&1
ls gpurun_out
