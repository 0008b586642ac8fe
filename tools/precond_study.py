"""configs[2]: preconditioner study on ~100k blocks — block-Jacobi vs SSOR-AI vs
ILU(0): iterations, construction ms, application ms, total solve ms; the B200
analog of the paper's Table I.  One JSON line per preconditioner."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
if os.environ.get("DDA_LIB_PATH"):          # A/B against another build of the library
    dda.LIB_PATH = os.environ["DDA_LIB_PATH"]
from synth import make_slope, preset


def ev_time(fn, reps=1):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); a.record()
    for _ in range(reps):
        fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000
    P = make_slope(preset("precond") if n == 100_000 else preset(n, seed=1003))
    t = dda.problem_to_device(P)
    F = t["F"]
    r = torch.randn_like(F)
    for pc in ("bj", "ssor_ai", "ilu0"):
        K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
        if pc == "ilu0":
            first = ev_time(lambda: K.precond_apply(r, "ilu0"))          # analysis + factor + one apply
            apply_ms = ev_time(lambda: K.precond_apply(r, "ilu0"), 5)
            construct = first - apply_ms
        else:   # warm (the first call also allocates the factor arrays), then the median of repeated setups
            K.bj_setup()
            construct = sorted(ev_time(lambda: K.bj_setup()) for _ in range(5))[2]
            apply_ms = ev_time(lambda: K.precond_apply(r, pc), 20)
        K.pcg_solve(F, precond=pc)                                       # warm (graph instantiation)
        res = {}
        solve = ev_time(lambda: res.setdefault("o", K.pcg_solve(F, precond=pc)))
        d, it, rr, st = res["o"]
        print(json.dumps({"blocks": K.n, "precond": pc, "iterations": it, "construction_ms": construct,
                          "application_ms": apply_ms, "solve_ms": solve, "ms_per_iteration": solve / max(it, 1),
                          "true_rel_res": rr, "status": st,
                          "paper_table1_k20_k40": {"bj": [275, 0.059, 0.011, 60330 / 1000],
                                                   "ssor_ai": [141, 0.208, 0.118, 62830 / 1000],
                                                   "ilu0": [93, 31.465, 7.269, 873787 / 1000]}[pc]}), flush=True)
        K.free()


if __name__ == "__main__":
    main()
