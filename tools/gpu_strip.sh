# single-reduction loop: parity tests + crossover sizes
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -k "not fullsize" -m gpu -x -q > gpurun_out/pytest_cg1.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_cg1.log
for n in 50000 70000; do
timeout 300 python tools/ab_env.py "DDA_SCALED_CG1=0;DDA_SCALED_CG1=1" $n 5 2>&1 | tail -1 >> gpurun_out/ab_cg1_sizes.jsonl
done
