timeout 600 python tools/precond_study.py 100000 > gpurun_out/ps_100k.jsonl 2>&1
DDA_PCG_ENGINE=graph timeout 600 python tools/precond_study.py 100000 > gpurun_out/ps_100k_graph.jsonl 2>&1
timeout 900 python tools/precond_study.py 1000000 > gpurun_out/ps_1m.jsonl 2>&1
for f in ps_100k ps_100k_graph ps_1m; do echo "== $f"; cut -c1-260 gpurun_out/$f.jsonl; done
