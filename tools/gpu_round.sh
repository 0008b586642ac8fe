# One GPU round: parity tests, smoke, bench line, ncu launch list, solve traffic, full-set captures, loop timeline.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; cat gpurun_out/bench.json
timeout 600 python bench.py --impl reference --steps 1 --warmup 0 > gpurun_out/bench_ref.json 2>&1; tail -1 gpurun_out/bench_ref.json
timeout 300 python tools/trace_loop.py 1000000 > gpurun_out/loop_trace.json 2>&1; cut -c1-400 gpurun_out/loop_trace.json
timeout 900 ncu --graph-profiling graph --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --spmv-reps 3 > gpurun_out/bench_ncu.log 2>&1; echo "ncu launches rc=$?"
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --csv --log-file gpurun_out/solve_traffic.csv python tools/prof_case.py --spmv 1 --pcg-maxit 10000 > gpurun_out/prof_case.log 2>&1; echo "ncu traffic rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_sp_loop --launch-count 1 -o gpurun_out/sp_loop python tools/prof_case.py --spmv 0 --pcg-maxit 40 > gpurun_out/prof_loop.log 2>&1; echo "ncu loop rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_spmv --launch-skip 3 --launch-count 1 -o gpurun_out/spmv_std python tools/prof_case.py --spmv 5 --pcg-maxit 1 > gpurun_out/prof_std.log 2>&1; echo "ncu std rc=$?"
