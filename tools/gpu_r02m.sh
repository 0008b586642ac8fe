python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python tools/time_next.py contacts,openclose,reorder 1000000 > gpurun_out/time_next.jsonl 2> gpurun_out/time_next.err; echo "rc=$?"; cat gpurun_out/time_next.jsonl; tail -3 gpurun_out/time_next.err
