python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "ilu0 or precond_apply or trend" > gpurun_out/pytest_p.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_p.log
python tools/precond_study.py 100000 > gpurun_out/precond_100k.jsonl 2>&1; cat gpurun_out/precond_100k.jsonl
python tools/precond_study.py 1000000 > gpurun_out/precond_1m.jsonl 2>&1; cat gpurun_out/precond_1m.jsonl
