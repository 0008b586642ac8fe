set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 300 python tools/scale_cmp.py 1000000 5 > gpurun_out/scale_cmp.json 2>&1; tail -3 gpurun_out/scale_cmp.json
timeout 300 python tools/scale_cmp.py 4000 5 >> gpurun_out/scale_cmp.json 2>&1; tail -1 gpurun_out/scale_cmp.json
