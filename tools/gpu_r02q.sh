python -c "import __graft_entry__ as g; g.build()"
python tools/ab_flag.py dda__set_sp_l1 2,0 1000000 8 > gpurun_out/ab_l1b.json 2>&1; cat gpurun_out/ab_l1b.json
python tools/ab_flag.py dda__set_sp_l1 0,2 1000000 8 > gpurun_out/ab_l1c.json 2>&1; cat gpurun_out/ab_l1c.json
