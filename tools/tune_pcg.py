"""PCG kernel variant sweep (tuning aid): ms per iteration at a given size."""
import json, os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

def child(blocks, pc):
    import torch
    import paper_conf_ipps_xiaohmxw17_b200 as dda
    from synth import make_slope, preset
    P = make_slope(preset(blocks, seed=1005))
    t = dda.problem_to_device(P)
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    K.bj_setup()
    K.pcg_solve(t["F"], precond=pc)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    res = []
    for _ in range(3):
        torch.cuda.synchronize(); a.record()
        d, it, rr, st = K.pcg_solve(t["F"], precond=pc)
        b.record(); torch.cuda.synchronize()
        res.append(a.elapsed_time(b))
    ms = min(res)
    print(json.dumps({"variant": os.environ.get("DDA_PCG_VARIANT"), "blocks": K.n, "pc": pc, "iters": it,
                      "ms": ms, "us_per_iter": 1000 * ms / it, "rel_res": rr}), flush=True)

if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "child":
        child(int(sys.argv[2]), sys.argv[3]); sys.exit(0)
    for n in [int(s) for s in os.environ.get("SIZES", "1000000").split(",")]:
        for pc in os.environ.get("PCS", "bj").split(","):
            for v in range(int(os.environ.get("NVAR", "3"))):
                subprocess.run([sys.executable, __file__, "child", str(n), pc], env=dict(os.environ, DDA_PCG_VARIANT=str(v)))
