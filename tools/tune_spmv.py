"""SpMV variant sweep (tuning aid, not a benchmark): times dda_spmv for each
compiled variant (DDA_SPMV_VARIANT) at several sizes, hot back-to-back."""
import json, os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

def child(blocks, reps, shuffle):
    import torch
    import paper_conf_ipps_xiaohmxw17_b200 as dda
    from synth import make_slope, preset
    P = make_slope(preset(blocks, seed=1005, shuffle=shuffle))
    t = dda.problem_to_device(P)
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    x = torch.rand(6 * K.n, dtype=torch.float64, device="cuda"); y = torch.empty_like(x)
    for _ in range(3): K.spmv(x, y)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); a.record()
    for _ in range(reps): K.spmv(x, y)
    b.record(); torch.cuda.synchronize()
    ms = a.elapsed_time(b) / reps
    u = K.nnzb / K.n
    gbs = K.n * (392 + 300 * u) / (ms * 1e-3) / 1e9
    print(json.dumps({"variant": os.environ.get("DDA_SPMV_VARIANT"), "blocks": K.n, "shuffle": shuffle,
                      "ms": ms, "gbs": gbs, "frac": gbs / 6552.0}), flush=True)

if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "child":
        child(int(sys.argv[2]), int(sys.argv[3]), sys.argv[4] == "1")
        sys.exit(0)
    nvar = int(os.environ.get("NVAR", "6"))
    sizes = [int(s) for s in os.environ.get("SIZES", "1000000").split(",")]
    for n in sizes:
        for v in range(nvar):
            env = dict(os.environ, DDA_SPMV_VARIANT=str(v))
            subprocess.run([sys.executable, __file__, "child", str(n), "50", os.environ.get("SHUF", "0")], env=env)
