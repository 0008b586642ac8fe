nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv
python tools/ab_flag.py dda__set_dyn_tail 0,1 1000000 6 > gpurun_out/ab_dyn.json 2>&1; cat gpurun_out/ab_dyn.json
python tools/trace_loop.py 1000000 > gpurun_out/loop_trace_dyn.json 2>&1; cut -c1-600 gpurun_out/loop_trace_dyn.json
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_sp_loop --launch-count 1 -o gpurun_out/sp_loop_r02 python tools/prof_case.py --spmv 0 --pcg-maxit 40 > gpurun_out/prof_loop.log 2>&1; echo "ncu loop rc=$?"
