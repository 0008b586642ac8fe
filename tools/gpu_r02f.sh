nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv
python tools/ab_flag.py dda__set_sp_variant 0,1,2,3 1000000 5 > gpurun_out/ab_sp.json 2>&1; cat gpurun_out/ab_sp.json
