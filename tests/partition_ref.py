"""TEST HELPER — host (numpy) reference of the block-row partition.

The product builds partitions on the device behind the C ABI (dda_build_matrix_dist,
csrc/dist_build.cu); this module is the independent host-side statement of the same
selection / numbering / exchange plan that the tests compare it with, and the
distributed-PCG emulation of tests/test_partition.py runs on it.

The paper is single-GPU; multi-GPU is its future work.  The path
shards by block rows: rank p owns the contiguous rows [r_p, r_{p+1}).  Each
rank assembles an ordinary local matrix (dda_build_matrix) from the springs
that touch its rows, in a LOCAL numbering:

    own rows   0 .. n_own-1            (global r_p .. r_{p+1}-1, same order)
    halo rows  n_own .. n_own+n_halo-1 (remote endpoints of those springs),
               grouped by owning rank (ascending), global order inside a group

Because every spring touching an own row is present, the local rows 0..n_own-1
of the local matrix are exactly the global rows (D_i, all couplings V_ij and
V_ki) under that relabelling; halo rows are only read as x values.  One halo
exchange per SpMV fills x[n_own:] — the segment received from peer q is
contiguous (halo grouped by owner), so it is received in place; the segment
sent to q lists the own rows that q holds as halo, in q's order.

(Host logic, numpy; the product equivalent is dda_build_matrix_dist.)
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


def row_bounds(n: int, nranks: int, weights: np.ndarray | None = None) -> np.ndarray:
    """Contiguous balanced row ranges [b[p], b[p+1]); balanced by `weights`
    (e.g. 1 + blocks per row) if given, else by row count."""
    if nranks < 1 or n < nranks:
        raise ValueError("need 1 <= nranks <= n")
    if weights is None:
        return np.array([(p * n) // nranks for p in range(nranks + 1)], dtype=np.int64)
    c = np.concatenate([[0], np.cumsum(np.asarray(weights, dtype=np.float64))])
    tgt = c[-1] * np.arange(nranks + 1) / nranks
    b = np.searchsorted(c, tgt, side="left").astype(np.int64)
    b[0], b[-1] = 0, n
    for p in range(1, nranks + 1):          # strictly increasing (each rank >= 1 row)
        b[p] = max(b[p], b[p - 1] + 1)
    for p in range(nranks - 1, 0, -1):
        b[p] = min(b[p], b[p + 1] - 1)
    return b


def owner_of(ids: np.ndarray, bounds: np.ndarray) -> np.ndarray:
    return np.searchsorted(bounds, ids, side="right") - 1


@dataclass
class LocalProblem:
    rank: int
    nranks: int
    r0: int
    r1: int
    n_own: int
    n_halo: int
    halo_global: np.ndarray     # [n_halo] global ids of halo rows (local id n_own + k)
    kdiag: np.ndarray           # [n_own + n_halo, 6, 6]; zeros for halo rows
    bi: np.ndarray              # local ids, int32
    bj: np.ndarray
    pen: np.ndarray
    e: np.ndarray
    g: np.ndarray
    F: np.ndarray               # [6 n_own]
    send_counts: np.ndarray     # [nranks] rows sent to each peer
    send_idx: np.ndarray        # local ids of the rows sent, concatenated by peer
    recv_counts: np.ndarray     # [nranks] halo rows received from each peer (contiguous)

    @property
    def n_local(self) -> int:
        return self.n_own + self.n_halo


def local_problem(n: int, kdiag, bi, bj, pen, e, g, F, bounds: np.ndarray, rank: int) -> LocalProblem:
    nranks = len(bounds) - 1
    r0, r1 = int(bounds[rank]), int(bounds[rank + 1])
    bi = np.asarray(bi); bj = np.asarray(bj)
    own_i = (bi >= r0) & (bi < r1)
    own_j = (bj >= r0) & (bj < r1)
    sel = np.nonzero(own_i | own_j)[0]                 # springs touching an own row, in spring order
    sbi, sbj = bi[sel].astype(np.int64), bj[sel].astype(np.int64)
    remote = np.concatenate([sbi[~own_i[sel]], sbj[~own_j[sel]]])
    halo = np.unique(remote)                           # global order == grouped by owner (contiguous ranges)
    n_own = r1 - r0

    def to_local(x):
        out = x - r0
        m = (x < r0) | (x >= r1)
        out[m] = n_own + np.searchsorted(halo, x[m])
        return out.astype(np.int32)

    lbi, lbj = to_local(sbi), to_local(sbj)
    kd = np.zeros((n_own + halo.size, 6, 6))
    kd[:n_own] = np.asarray(kdiag)[r0:r1]
    howner = owner_of(halo, bounds) if halo.size else np.zeros(0, np.int64)
    recv_counts = np.bincount(howner, minlength=nranks).astype(np.int32)
    # rows to send to q: own rows that share a spring with a row owned by q (q's halo order = global order)
    send_lists = []
    for q in range(nranks):
        if q == rank:
            send_lists.append(np.zeros(0, np.int64))
            continue
        q0, q1 = int(bounds[q]), int(bounds[q + 1])
        a = (sbi >= q0) & (sbi < q1)
        b = (sbj >= q0) & (sbj < q1)
        rows = np.unique(np.concatenate([sbj[a], sbi[b]]))
        rows = rows[(rows >= r0) & (rows < r1)]
        send_lists.append(rows - r0)
    send_counts = np.array([s.size for s in send_lists], np.int32)
    send_idx = (np.concatenate(send_lists) if send_lists else np.zeros(0)).astype(np.int32)
    return LocalProblem(rank=rank, nranks=nranks, r0=r0, r1=r1, n_own=n_own, n_halo=int(halo.size),
                        halo_global=halo.astype(np.int64), kdiag=kd, bi=lbi, bj=lbj,
                        pen=np.ascontiguousarray(np.asarray(pen)[sel]),
                        e=np.ascontiguousarray(np.asarray(e)[sel]), g=np.ascontiguousarray(np.asarray(g)[sel]),
                        F=np.ascontiguousarray(np.asarray(F).reshape(-1, 6)[r0:r1].reshape(-1)),
                        send_counts=send_counts, send_idx=send_idx, recv_counts=recv_counts)


def local_from_slope(P, bounds, rank) -> LocalProblem:
    return local_problem(P.n, P.kdiag, P.bi, P.bj, P.pen, P.e, P.g, P.F, bounds, rank)
