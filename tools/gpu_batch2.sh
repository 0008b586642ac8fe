set -x
nvidia-smi --query-gpu=name,memory.used,clocks.sm,power.draw,temperature.gpu --format=csv
timeout 400 python bench.py --no-cpu > gpurun_out/bench_s5.json 2> gpurun_out/bench_s5.err
timeout 300 python tools/time_step.py > gpurun_out/time_step.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_g_spmv --launch-skip 2 --launch-count 1 -o gpurun_out/spmv_sc python tools/prof_phases.py 1000000 1 > gpurun_out/prof_spmv.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_s_update --launch-skip 2 --launch-count 1 -o gpurun_out/upd_sc python tools/prof_phases.py 1000000 1 > gpurun_out/prof_upd.log 2>&1
timeout 400 python bench.py --no-cpu > gpurun_out/bench_s6.json 2> gpurun_out/bench_s6.err
