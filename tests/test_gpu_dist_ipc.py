"""§8(e): the IPC transport with real processes (beyond the paper: multi-GPU is its future work).

Two (or three) processes share the one GPU of the test box, one partition each: every rank builds its
partition behind the C ABI (dda_build_matrix_dist), exports its CUDA IPC handles, the blobs are
exchanged over a gloo process group (the caller's channel), and the block-Jacobi PCG runs as v7: one
persistent cooperative kernel per process, halo rows read in place from the peers' mapped arrays,
every reduction a fixed-order one-shot sum through rank 0's mapped slot sets.  The processes'
kernels share the GPU by time slicing, so this checks the protocol, not the speed.  Rank 0 gathers
the solution; the test compares it with the oracle (reading Z17).  A warm start and a rebuilt partition
(the next step's matrix, re-attached into the mapped buffers) are checked too.
"""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

pytestmark = pytest.mark.gpu

WORKER = r"""
import json, os, sys
sys.path.insert(0, os.environ["DDA_ROOT"])
import numpy as np
import torch
import torch.distributed as dist
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset

rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
dist.init_process_group("gloo", init_method="tcp://127.0.0.1:" + os.environ["PORT"], rank=rank, world_size=world)
torch.cuda.set_device(0)
P = make_slope(preset(os.environ["CASE"]))
t = dda.problem_to_device(P)
b = dda.row_bounds(P.n, world)
r0, r1 = int(b[rank]), int(b[rank + 1])
comm = dda.Comm.ipc(world, rank)
K = comm.build_matrix_dist(0, P.n, b, t["kdiag"][r0:r1].contiguous(), t["bi"], t["bj"], t["pen"], t["e"], t["g"])
blobs = [None] * world
dist.all_gather_object(blobs, comm.ipc_export())
comm.ipc_import(blobs)
F = t["F"][6 * r0:6 * r1].contiguous()
out = {}
ds, it, rr, st = comm.pcg_solve([F], tol=1e-10, precond="bj")
out["cold"] = (it, rr, st)
d = ds[0].cpu().numpy()
# warm start from the solution (every rank's own rows): at most one iteration
ds2, it2, rr2, st2 = comm.pcg_solve([F], d0s=[ds[0].clone()], tol=1e-10, precond="bj")
out["warm"] = (it2, rr2, st2)
# the next step's rebuilt partition re-attaches into the mapped buffers (same plan): same solve
K = comm.build_matrix_dist(0, P.n, b, t["kdiag"][r0:r1].contiguous(), t["bi"], t["bj"], t["pen"], t["e"], t["g"])
ds3, it3, rr3, st3 = comm.pcg_solve([F], tol=1e-10, precond="bj")
out["rebuilt_same"] = bool(it3 == it and torch.equal(ds3[0], ds[0]))
parts = [None] * world
dist.all_gather_object(parts, d.tolist())
if rank == 0:
    out["d"] = [x for p in parts for x in p]
    with open(os.environ["OUT"], "w") as f:
        json.dump(out, f)
dist.barrier()
comm.free()
"""


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("case_name,world", [("tiny", 2), ("paper", 2), ("paper", 3)])
def test_ipc_processes_pcg(case_name, world, tmp_path):
    import oracle
    from synth import make_slope, preset
    out = tmp_path / "out.json"
    port = str(_free_port())
    env_base = dict(os.environ, DDA_ROOT=ROOT, PORT=port, CASE=case_name, OUT=str(out), WORLD_SIZE=str(world),
                    MASTER_ADDR="127.0.0.1")
    procs = [subprocess.Popen([sys.executable, "-c", WORKER], env=dict(env_base, RANK=str(r)),
                              stdout=subprocess.PIPE, stderr=subprocess.STDOUT) for r in range(world)]
    logs = []
    try:
        for p in procs:
            o, _ = p.communicate(timeout=600)
            logs.append(o.decode(errors="replace")[-3000:])
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    assert all(p.returncode == 0 for p in procs), "\n----\n".join(logs)
    res = json.loads(out.read_text())
    it, rr, st = res["cold"]
    assert st == 0 and rr <= 1.01e-10, res["cold"]
    assert res["warm"][2] == 0 and res["warm"][0] <= 1, res["warm"]
    assert res["rebuilt_same"]
    P = make_slope(preset(case_name))
    O = oracle.assemble(P)
    do, ito, rro, sto = O.pcg(P.F, tol=1e-10, precond="bj")
    assert abs(it - ito) <= max(2, int(0.01 * ito)), (it, ito)
    dm, itm, _, _ = O.pcg(P.F, tol=1e-300, maxit=it, precond="bj")
    d = np.array(res["d"])
    assert np.linalg.norm(d - dm) / np.linalg.norm(dm) <= 1e-9
