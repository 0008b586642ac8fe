python -c "import __graft_entry__ as g; g.build()"
timeout 600 python tools/open_close.py 1000000 4 > gpurun_out/open_close.json 2>&1; cut -c1-900 gpurun_out/open_close.json
timeout 900 python tools/time_next.py openclose 1000000 > gpurun_out/time_next_oc.jsonl 2>&1; cat gpurun_out/time_next_oc.jsonl
