python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests/test_gpu_reorder.py tests/test_gpu_hsbcsr.py -q > gpurun_out/pytest_g.log 2>&1; echo "pytest rc=$?"; tail -25 gpurun_out/pytest_g.log
python tools/hsbcsr_cmp.py > gpurun_out/hsbcsr_cmp.jsonl 2>&1; cat gpurun_out/hsbcsr_cmp.jsonl
