"""NEXT-3 measurement: dda_detect_contacts + dda_contact_springs on the configs[4] slope geometry
(1M blocks, 4M vertices), CUDA events, and the same pipeline feeding dda_build_matrix.  One JSON line."""
import json, os, sys, statistics, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
d0 = float(sys.argv[2]) if len(sys.argv) > 2 else 0.2
P = make_slope(preset(n, seed=1005))
vptr = torch.from_numpy((4 * np.arange(P.n + 1)).astype(np.int32)).cuda()
vxy = torch.from_numpy(P.verts.reshape(-1, 2).copy()).cuda()
cxy = torch.from_numpy(P.centroid.copy()).cuda()
kd = torch.from_numpy(P.kdiag).cuda()
det, spr, bld = [], [], []
for rep in range(6):
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    c = torch.cuda.Event(enable_timing=True); d = torch.cuda.Event(enable_timing=True)
    a.record()
    C = dda.detect_contacts(vptr, vxy, d0)
    b.record()
    S = C.springs(cxy, 40.0, 0.4)
    c.record()
    K = dda.build_matrix(kd, S["bi"], S["bj"], S["pen"], S["e"], S["g"])
    d.record()
    torch.cuda.synchronize()
    if rep:
        det.append(a.elapsed_time(b)); spr.append(b.elapsed_time(c)); bld.append(c.elapsed_time(d))
    info = (C.count, C.n_ve, C.n_pairs, K.nnzb)
    K.free(); C.free()
V = 4 * P.n
print(json.dumps({"n_blocks": P.n, "vertices": V, "d0": d0, "pairs": info[2], "records": info[0], "ve": info[1],
                  "springs": 2 * info[1], "nnzb": info[3], "generator_contacts": P.n_contacts,
                  "detect_ms": statistics.median(det), "springs_ms": statistics.median(spr),
                  "build_ms": statistics.median(bld),
                  "detect_blocks_per_s": P.n / (statistics.median(det) * 1e-3),
                  "note": "detect includes its three host read-backs of counts (stream syncs)"}), flush=True)
