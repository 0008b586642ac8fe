"""The oracle's own full BJ-PCG solve of bench.py's workload (configs[4] at N = 1, seed 1005),
timed end to end on ONE pinned host core.  Calls only synth/ and oracle/ (no CUDA path).

Writes profiles/r02_oracle_1m.json: the iteration count and relative residual of the oracle's
solve to 1e-10 on that exact system (the count bench.py's cpu_baseline and --impl reference legs
multiply their measured per-iteration time by), and the measured wall times of each part.

usage: python tools/oracle_1m.py [n_blocks] [out.json]
"""
import hashlib
import json
import os
import platform
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np

import oracle
from synth import make_slope, preset


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor() or "unknown"


def fingerprint(P):
    h = hashlib.sha256()
    for a in (P.bi, P.bj, P.pen, P.F):
        h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()[:16]


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
    out = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "profiles", "r02_oracle_1m.json")
    core = sorted(os.sched_getaffinity(0))[0]
    os.sched_setaffinity(0, {core})
    P = make_slope(preset(n, seed=1005))
    t0 = time.perf_counter()
    M = oracle.assemble(P)
    M.full_csr()
    t1 = time.perf_counter()
    d, it, rr, st = M.pcg(P.F, tol=1e-10, maxit=10000, precond="bj")
    t2 = time.perf_counter()
    rec = {"n_blocks": int(P.n), "springs": int(P.m), "fingerprint": fingerprint(P), "precond": "bj", "tol": 1e-10,
           "oracle_iters": int(it), "oracle_rel_res": float(rr), "status": int(st),
           "seconds": {"assemble_expand": t1 - t0, "pcg": t2 - t1, "total": t2 - t0},
           "cores": 1, "pinned_core": core, "cpu_model": cpu_model(),
           "script": "tools/oracle_1m.py (synth + oracle only)"}
    with open(out, "w") as f:
        json.dump(rec, f, indent=1)
    print(json.dumps(rec))


if __name__ == "__main__":
    main()
