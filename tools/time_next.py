"""Measurements of the NEXT rows at the configs[4] size (1M blocks), one JSON line each:
  contacts   NEXT-3: dda_detect_contacts, dda_classify_contacts (angle judgment, VV1 / VV2),
             dda_contact_springs on the slope's polygons (d0 = 0.2 h, sin_tol 0.35)
  openclose  NEXT-4: dda_contact_init, then loop 3 (dda_open_close: value-only re-assembly +
             gap load + warm-started BJ-PCG + interpenetration check) to its fixed point under
             self-weight; the check and load kernels timed alone with their algorithmic bytes
  reorder    NEXT-2: dda_spmv on a randomly numbered 1M slope, plain vs dda_build_matrix_reordered
Tuning / measurement aid."""
import json, os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
try:
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("hbm_gbs", 6552.0)
except OSError:
    peak = 6552.0


def timed(fn, reps=5):
    fn(); torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


what = sys.argv[1].split(",") if len(sys.argv) > 1 else ["contacts", "openclose", "reorder"]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1_000_000
P = make_slope(preset(n, seed=1005))
vptr = torch.from_numpy((4 * np.arange(P.n + 1)).astype(np.int32)).cuda()
vxy = torch.from_numpy(np.ascontiguousarray(P.verts.reshape(-1, 2))).cuda()
cxy = torch.from_numpy(np.ascontiguousarray(P.centroid)).cuda()

if "contacts" in what:
    t_det = timed(lambda: dda.detect_contacts(vptr, vxy, 0.2).free())

    def det_cls():
        C = dda.detect_contacts(vptr, vxy, 0.2)
        C.classify(0.35)
        C.free()
    t_cls = timed(det_cls) - t_det
    C = dda.detect_contacts(vptr, vxy, 0.2)
    n_rec = C.count
    C.classify(0.35)
    t_spr = timed(lambda: C.springs(cxy, 40.0, 0.4))
    print(json.dumps({"row": "NEXT-3", "blocks": P.n, "records": n_rec, "kept": C.count, "ve": C.n_ve,
                      "vv1": C.n_vv1, "vv2": C.n_vv2, "detect_ms": t_det, "classify_ms": t_cls,
                      "springs_ms": t_spr, "springs": 2 * C.count}), flush=True)
    C.free()

if "openclose" in what:
    C = dda.detect_contacts(vptr, vxy, 0.2)
    C.classify(0.35)
    sp = C.springs(cxy, 40.0, 0.4)
    state0 = C.init_states()
    V = P.verts
    area = 0.5 * np.abs(np.sum(V[:, :, 0] * np.roll(V[:, :, 1], -1, 1) - np.roll(V[:, :, 0], -1, 1) * V[:, :, 1], 1))
    Fh = np.zeros((P.n, 6))
    Fh[:, 1] = -area
    F = torch.from_numpy(Fh.reshape(-1)).cuda()
    kd = torch.from_numpy(P.kdiag).cuda()
    K = dda.build_matrix(kd, sp["bi"], sp["bj"], sp["pen"], sp["e"], sp["g"])
    st = state0.clone()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    d, st, pen, oc, pit, conv, rr = C.open_close(K, kd, F, sp, st, max_oc=40)
    b.record(); torch.cuda.synchronize()
    loop_ms = a.elapsed_time(b)
    counts = np.bincount(st.cpu().numpy(), minlength=3)
    # the check and the gap-load kernels alone (same d, states reset each time)
    old = st.clone()

    def chk():
        s2 = old.clone()
        C.check(d, sp, s2)
    t_chk = timed(chk)
    t_load = timed(lambda: C.loads(sp, pen, F))
    m = C.count
    # check: per contact e, g of two springs (4 x 48 B), two 48 B rows of d, gap, state r/w, pen and
    # category writes (2 x 8 + 4), sort keys / values (8); the category sort is extra
    b_chk = m * (4 * 48 + 2 * 48 + 8 + 8 + 16 + 4 + 8)
    # contact transfer to the next step (the same polygons moved by U(-0.01, 0.01) h)
    vxy2 = vxy + (torch.rand_like(vxy) - 0.5) * 0.02
    C2 = dda.detect_contacts(vptr, vxy2, 0.2)
    C2.classify(0.35)
    st2 = C2.init_states()
    t_tr = timed(lambda: C2.transfer_from(C, st, st2.clone()))
    matched = C2.transfer_from(C, st, st2)
    print(json.dumps({"row": "NEXT-3 transfer", "prev": C.count, "cur": C2.count, "matched": matched,
                      "transfer_ms": t_tr}), flush=True)
    print(json.dumps({"row": "NEXT-4", "blocks": P.n, "contacts": m, "converged": conv, "oc_iters": oc,
                      "pcg_iters_total": pit, "loop_ms": loop_ms, "final_states": {"open": int(counts[0]),
                      "slide": int(counts[1]), "lock": int(counts[2])}, "rel_res_last": rr,
                      "check_ms": t_chk, "check_algorithmic_gb": b_chk / 1e9,
                      "check_gbs": b_chk / (t_chk * 1e-3) / 1e9, "loads_ms": t_load}), flush=True)

if "reorder" in what:
    Ps = make_slope(preset(n, seed=1005, shuffle=True))
    t = dda.problem_to_device(Ps)
    Kp = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    import time
    h0 = time.perf_counter()
    Kr = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"], reorder=True)
    torch.cuda.synchronize()
    build_r_s = time.perf_counter() - h0
    x = torch.rand(6 * Ps.n, dtype=torch.float64, device="cuda")
    y = torch.empty_like(x)
    tp = timed(lambda: Kp.spmv(x, y), 20)
    tr = timed(lambda: Kr.spmv(x, y), 20)
    u = Kp.nnzb / Ps.n
    byt = Ps.n * (392 + 300 * u)
    sp_p = timed(lambda: Kp.pcg_solve(t["F"]), 2)
    sp_r = timed(lambda: Kr.pcg_solve(t["F"]), 2)
    print(json.dumps({"row": "NEXT-2", "blocks": Ps.n, "numbering": "random (seeded shuffle)",
                      "spmv_plain_us": 1000 * tp, "spmv_reordered_us": 1000 * tr,
                      "spmv_plain_frac_hbm": byt / (tp * 1e-3) / 1e9 / peak,
                      "spmv_reordered_frac_hbm": byt / (tr * 1e-3) / 1e9 / peak,
                      "pcg_plain_ms": sp_p, "pcg_reordered_ms": sp_r, "reordered_build_s": build_r_s}), flush=True)
