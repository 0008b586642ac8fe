"""Host logic of the multi-GPU path, on CPU: the block-row
partition, the halo plan (checked across ranks with a world_size-2 gloo group),
bit-exactness of the local assemblies' own rows against the global oracle, and
a distributed PCG emulation (numpy SpMV on local matrices + gloo halo exchange
and allreduce) that must match the global oracle's iteration count."""
import os
import socket

import numpy as np
import pytest
import scipy.sparse as sp
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from partition_ref import row_bounds, local_from_slope, owner_of
from synth import make_slope, preset


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _problem():
    return make_slope(preset(2000, seed=1042))


def test_row_bounds_balanced():
    b = row_bounds(1000, 4)
    assert b.tolist() == [0, 250, 500, 750, 1000]
    w = np.ones(1000); w[:500] = 3
    bw = row_bounds(1000, 2, w)
    assert 0 < bw[1] < 500 and bw[-1] == 1000
    assert (np.diff(row_bounds(10, 10)) == 1).all()


@pytest.mark.parametrize("nranks", [2, 3])
def test_local_rows_bit_exact(nranks):
    P = _problem()
    O = oracle.assemble(P)
    G = O.export()
    b = row_bounds(P.n, nranks)
    for rank in range(nranks):
        lp = local_from_slope(P, b, rank)
        L = oracle.OracleMatrix(lp.n_local, lp.kdiag, lp.bi, lp.bj, lp.pen, lp.e, lp.g).export()
        glob = np.concatenate([np.arange(lp.r0, lp.r1), lp.halo_global])       # local -> global id
        # diagonal blocks of own rows are identical
        assert np.array_equal(L.diag[:lp.n_own], G.diag[lp.r0:lp.r1])
        # every coupling of an own row, both directions, is identical to the global block
        for i in range(lp.n_own):
            gi = lp.r0 + i
            for u in range(L.row_ptr[i], L.row_ptr[i + 1]):
                gj = glob[L.col_idx[u]]
                blk = L.upper[u]
                a, c = (gi, gj) if gi < gj else (gj, gi)
                gu = np.nonzero((G.col_idx[G.row_ptr[a]:G.row_ptr[a + 1]] == c))[0]
                assert gu.size == 1
                gblk = G.upper[G.row_ptr[a] + gu[0]]
                assert np.array_equal(blk, gblk if gi < gj else gblk.T)
            for t in range(L.low_ptr[i], L.low_ptr[i + 1]):                      # local lower = own rows only
                assert L.low_row[t] < lp.n_own
        # halo grouped by owner, contiguous, counts match
        own = owner_of(lp.halo_global, b)
        assert (np.diff(own) >= 0).all()
        assert np.bincount(own, minlength=nranks).tolist() == lp.recv_counts.tolist()


def _worker(rank, world, port, outq):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        P = _problem()
        b = row_bounds(P.n, world)
        lp = local_from_slope(P, b, rank)
        # --- halo plan consistency: what I send to q is what q receives from me
        sc = torch.tensor(lp.send_counts, dtype=torch.int64)
        rc_of_peers = [torch.zeros(world, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(rc_of_peers, torch.tensor(lp.recv_counts, dtype=torch.int64))
        for q in range(world):
            assert int(sc[q]) == int(rc_of_peers[q][rank])
        # global ids sent to q == q's halo ids from me
        halos = [None] * world
        dist.all_gather_object(halos, (lp.halo_global.tolist(), b.tolist()))
        off = np.concatenate([[0], np.cumsum(lp.send_counts)])
        for q in range(world):
            if q == rank:
                continue
            sent = (lp.send_idx[off[q]:off[q + 1]] + lp.r0).tolist()
            qh = np.array(halos[q][0], np.int64)
            mine = qh[(qh >= lp.r0) & (qh < lp.r1)].tolist()
            assert sent == mine
        # --- distributed PCG-BJ emulation: local numpy SpMV + gloo halo + allreduce
        L = oracle.OracleMatrix(lp.n_local, lp.kdiag, lp.bi, lp.bj, lp.pen, lp.e, lp.g)
        ip, ix, dv = L.full_csr()
        A = sp.csr_matrix((dv, ix, ip), shape=(6 * lp.n_local,) * 2)[: 6 * lp.n_own]
        Dinv = np.linalg.inv(L.export().diag[: lp.n_own])
        roff = np.concatenate([[0], np.cumsum(lp.recv_counts)])

        def halo(xown):
            x = np.zeros(6 * lp.n_local)
            x[: 6 * lp.n_own] = xown
            reqs = []
            bufs = {}
            for q in range(world):
                if q == rank:
                    continue
                if lp.send_counts[q]:
                    idx = lp.send_idx[off[q]:off[q + 1]]
                    sbuf = torch.from_numpy(x.reshape(-1, 6)[idx].reshape(-1).copy())
                    reqs.append(dist.isend(sbuf, q))
                    bufs[("s", q)] = sbuf
                if lp.recv_counts[q]:
                    rbuf = torch.zeros(6 * int(lp.recv_counts[q]), dtype=torch.float64)
                    reqs.append(dist.irecv(rbuf, q))
                    bufs[("r", q)] = rbuf
            for r in reqs:
                r.wait()
            for q in range(world):
                if ("r", q) in bufs:
                    a = 6 * (lp.n_own + roff[q])
                    x[a:a + bufs[("r", q)].numel()] = bufs[("r", q)].numpy()
            return x

        def allsum(*v):
            t = torch.tensor(v, dtype=torch.float64)
            dist.all_reduce(t)
            return t.tolist()

        F = lp.F
        d = np.zeros_like(F)
        r = F.copy()
        z = np.einsum("bij,bj->bi", Dinv, r.reshape(-1, 6)).ravel()
        p = z.copy()
        FF, rho = allsum(F @ F, r @ z)
        it = 0
        for k in range(5000):
            qv = A @ halo(p)
            (sigma,) = allsum(p @ qv)
            alpha = rho / sigma
            d += alpha * p
            r -= alpha * qv
            z = np.einsum("bij,bj->bi", Dinv, r.reshape(-1, 6)).ravel()
            rr, rz = allsum(r @ r, r @ z)
            it = k + 1
            if np.sqrt(rr) <= 1e-10 * np.sqrt(FF):
                break
            p = z + (rz / rho) * p
            rho = rz
        outq.put((rank, it, lp.r0, d))
    finally:
        dist.destroy_process_group()


def test_distributed_pcg_emulation_gloo():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    P = _problem()
    O = oracle.assemble(P)
    d_ref, it_ref, rr_ref, st = O.pcg(P.F, tol=1e-10, precond="bj")
    its = {r: it for r, it, _, _ in res}
    assert its[0] == its[1]
    assert abs(its[0] - it_ref) <= max(2, int(0.01 * it_ref))
    d = np.zeros(6 * P.n)
    for _, _, r0, dl in res:
        d[6 * r0: 6 * r0 + dl.size] = dl
    assert np.linalg.norm(d - d_ref) <= 1e-7 * np.linalg.norm(d_ref)
