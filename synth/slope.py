"""Jittered-brick slope generator: the synthetic stand-in for the paper's slope models.

The paper's models (case 1: a realistic slope of 4361 blocks with 5 block
materials; case 2: a rock fall) are not available, so
the inputs of the solve K·d = F are drawn from a seeded 2-D blocky slope with
the same structure:

* blocks are quadrilateral bricks laid in running bond (courses of height h,
  bricks of length 2h, odd courses offset by h), cut by a 45-degree slope face
  on the right; every vertex is jittered by U(-0.08h, 0.08h);
* each block has the six DDA unknowns (u0, v0, r0, ex, ey, gxy) — Shi's
  first-order displacement function (external: Shi 1988, ref [1] P:292);
* every pair of touching blocks gets two vertex-edge contacts at the ends of
  their shared edge (the VE class of P:70-72); a contact is "lock" with
  probability 0.7 (normal + shear spring) or "slide" (normal spring only);
  open contacts are abandoned and never emitted;
* a spring s between vertex block i and edge block j is (i, j, p, e, g):
  its contribution to K is [e; g] p [e; g]^T over the two blocks, i.e. it adds
  to a_ii, a_jj, a_ij and a_ji;
* the per-block diagonal terms Kd_i are elastic + inertia + fixed points
  (Table II P:250 "diagonal matrix building"), computed here
  because the ABI takes them as an input.

Nothing in this module assembles, multiplies or solves: it has none of the
method's arithmetic.  DESIGN.md §3 states the recipe and its calibration.
"""
from __future__ import annotations

from dataclasses import dataclass, asdict
import math

import numpy as np

MATERIAL_E = (0.6, 0.8, 1.0, 1.2, 1.5)   # five block materials
NU = 0.25


@dataclass(frozen=True)
class SlopeConfig:
    base_bricks: int            # B0: full bricks (length 2h) in the base course
    courses: int                # number of courses (rows of bricks)
    slope: bool = True          # 45-degree slope face cutting the right end
    h: float = 1.0              # course height
    jitter: float = 0.08        # vertex jitter as a fraction of h
    lock_prob: float = 0.7      # P(lock) -> 2 springs, else slide -> 1 spring
    penalty: float = 40.0       # reference normal penalty p_n0 = penalty * E_ref
    penalty_ratio: float = 30.0  # r: inertia c = p_n0 / (r * mean area); r=30 -> ~271 BJ iters at 10k (Table I: 275)
    fixed_ratio: float = 10.0   # fixed-point penalty = fixed_ratio * p_n0
    shuffle: bool = False       # seeded random relabelling of the blocks
    seed: int = 1000


@dataclass
class SlopeProblem:
    cfg: SlopeConfig
    n: int                      # number of blocks
    kdiag: np.ndarray           # [n, 6, 6] float64, symmetric
    bi: np.ndarray              # [m] int32, vertex block of the spring
    bj: np.ndarray              # [m] int32, edge block of the spring
    pen: np.ndarray             # [m] float64 >= 0
    e: np.ndarray               # [m, 6] float64
    g: np.ndarray               # [m, 6] float64
    F: np.ndarray               # [6n] float64 load vector
    course: np.ndarray          # [n] int32 course index of each block
    n_contacts: int
    # geometry (NEXT-3 inputs; block ids after the optional shuffle):
    verts: np.ndarray = None    # [n, 4, 2] jittered polygon vertices, counter-clockwise
    centroid: np.ndarray = None  # [n, 2]
    # the generator's own contacts (vertex cv = 4*i + k of block i against edge ce = 4*j + c of
    # block j, running to the next vertex of j; tau = edge ratio), before any spring permutation
    contacts: dict = None

    @property
    def m(self) -> int:
        return int(self.bi.shape[0])

    def summary(self) -> dict:
        return {"n_blocks": self.n, "dof": 6 * self.n, "contacts": self.n_contacts,
                "springs": self.m, "cfg": asdict(self.cfg)}


# --------------------------------------------------------------------------------------
# presets: the five BASELINE.json configurations
# --------------------------------------------------------------------------------------

def _b0_for(n_target: int) -> int:
    # with courses == base_bricks and a 45-degree face, n ~= 0.75 * B0^2
    return max(2, int(round(math.sqrt(n_target / 0.75))))


PRESETS = {
    "tiny": 100,          # configs[0]: ~100 blocks, vs dense LDL^T
    "paper": 10_000,      # configs[1]: paper-scale slope
    "precond": 100_000,   # configs[2]: preconditioner study
    "1m": 1_000_000,      # configs[4]: 1M-block assembly + PCG
}


def preset(name_or_n, seed: int | None = None, **overrides) -> SlopeConfig:
    """SlopeConfig for a named preset or a target block count.

    Seeds follow SURVEY.md §8(d): config c uses 1000 + c; sweep point t uses 1040 + t.
    """
    if isinstance(name_or_n, str):
        n_target = PRESETS[name_or_n]
        default_seed = {"tiny": 1001, "paper": 1002, "precond": 1003, "1m": 1005}[name_or_n]
    else:
        n_target = int(name_or_n)
        default_seed = 1040
    b0 = _b0_for(n_target)
    kw = dict(base_bricks=b0, courses=b0, seed=default_seed if seed is None else seed)
    kw.update(overrides)
    return SlopeConfig(**kw)


# --------------------------------------------------------------------------------------
# geometry helpers (displacement function, external: Shi 1988)
# --------------------------------------------------------------------------------------

def _t_transpose_times(dx, dy, vx, vy):
    """T(P)^T v for the 2x6 first-order displacement matrix T at offset (dx, dy)
    from the block centroid; rows of T:
       [1, 0, -dy, dx, 0,  dy/2]
       [0, 1,  dx, 0,  dy, dx/2]
    Vectorised over leading dims; returns [..., 6]."""
    return np.stack([vx, vy, -dy * vx + dx * vy, dx * vx, dy * vy,
                     0.5 * dy * vx + 0.5 * dx * vy], axis=-1)


def _t_matrix(dx, dy):
    """T at offsets (dx, dy): returns [..., 2, 6]."""
    z = np.zeros_like(dx)
    o = np.ones_like(dx)
    r1 = np.stack([o, z, -dy, dx, z, 0.5 * dy], axis=-1)
    r2 = np.stack([z, o, dx, z, dy, 0.5 * dx], axis=-1)
    return np.stack([r1, r2], axis=-2)


def _layout(cfg: SlopeConfig):
    """Unperturbed running-bond bricks, course-major (bottom to top, left to right)."""
    h = cfg.h
    W = 2.0 * h * cfg.base_bricks
    lefts, xbs, xts, course = [], [], [], []
    for c in range(cfg.courses):
        y0, y1 = c * h, (c + 1) * h
        off = h if (c % 2) else 0.0
        edges = np.arange(off, W - 1e-9, 2.0 * h)
        if off > 0:
            edges = np.concatenate([[0.0], edges])
        edges = np.concatenate([edges, [W]])
        lo, hi = edges[:-1], edges[1:]
        if cfg.slope:
            xb = np.minimum(hi, W - y0)
            xt = np.minimum(hi, W - y1)
        else:
            xb, xt = hi.copy(), hi.copy()
        keep = (xt - lo) >= 0.5 * h
        if not keep.any():
            break
        lefts.append(lo[keep]); xbs.append(xb[keep]); xts.append(xt[keep])
        course.append(np.full(int(keep.sum()), c, dtype=np.int32))
    return lefts, xbs, xts, course


def _polygon_props(V):
    """Area and area-centroid of quads V[n,4,2] (CCW)."""
    x, y = V[..., 0], V[..., 1]
    xn, yn = np.roll(x, -1, axis=1), np.roll(y, -1, axis=1)
    cr = x * yn - xn * y
    A = 0.5 * cr.sum(axis=1)
    cx = ((x + xn) * cr).sum(axis=1) / (6.0 * A)
    cy = ((y + yn) * cr).sum(axis=1) / (6.0 * A)
    return A, cx, cy


def _inertia_integral(V, cx, cy, chunk=65536):
    """Exact  integral over the polygon of T^T T dA  (degree-2 integrand): fan
    triangulation from the centroid and the 3-edge-midpoint rule per triangle."""
    n = V.shape[0]
    out = np.empty((n, 6, 6))
    for s in range(0, n, chunk):
        Vs = V[s:s + chunk] - np.stack([cx[s:s + chunk], cy[s:s + chunk]], -1)[:, None, :]
        a = Vs
        b = np.roll(Vs, -1, axis=1)
        area = 0.5 * (a[..., 0] * b[..., 1] - a[..., 1] * b[..., 0])       # [k,4]
        pts = np.concatenate([0.5 * a, 0.5 * b, 0.5 * (a + b)], axis=1)   # [k,12,2]
        w = np.concatenate([area, area, area], axis=1) / 3.0               # [k,12]
        T = _t_matrix(pts[..., 0], pts[..., 1])                            # [k,12,2,6]
        out[s:s + chunk] = np.einsum("kpai,kpaj,kp->kij", T, T, w, optimize=True)
    return out


# --------------------------------------------------------------------------------------
# the generator
# --------------------------------------------------------------------------------------

def make_slope(cfg: SlopeConfig) -> SlopeProblem:
    rng = np.random.default_rng(cfg.seed)
    h = cfg.h
    lefts, xbs, xts, course_l = _layout(cfg)
    counts = [len(l) for l in lefts]
    starts = np.concatenate([[0], np.cumsum(counts)]).astype(np.int64)
    n = int(starts[-1])
    L = np.concatenate(lefts); XB = np.concatenate(xbs); XT = np.concatenate(xts)
    course = np.concatenate(course_l)
    y0 = course * h
    y1 = y0 + h
    V = np.empty((n, 4, 2))
    V[:, 0, 0], V[:, 0, 1] = L, y0
    V[:, 1, 0], V[:, 1, 1] = XB, y0
    V[:, 2, 0], V[:, 2, 1] = XT, y1
    V[:, 3, 0], V[:, 3, 1] = L, y1
    V += rng.uniform(-cfg.jitter * h, cfg.jitter * h, size=V.shape)
    area, cx, cy = _polygon_props(V)
    assert (area > 0).all()

    # ---------------- contacts: (vertex block i, vertex k) against (edge block j, P2 -> P3)
    ci, ck, cj, c2, c3 = [], [], [], [], []
    for c in range(len(counts)):
        ids = np.arange(starts[c], starts[c + 1])
        if ids.size >= 2:                       # horizontal neighbours a | b
            a, b = ids[:-1], ids[1:]
            ci.append(b); ck.append(np.full(a.size, 0)); cj.append(a)
            c2.append(np.full(a.size, 1)); c3.append(np.full(a.size, 2))
            ci.append(a); ck.append(np.full(a.size, 2)); cj.append(b)
            c2.append(np.full(a.size, 3)); c3.append(np.full(a.size, 0))
        if c + 1 < len(counts):                 # vertical: A in course c, B in c+1
            idb = np.arange(starts[c + 1], starts[c + 2])
            la, xta = L[ids], XT[ids]
            lb, xbb = L[idb], XB[idb]
            first = np.searchsorted(xbb, la, side="right")
            last = np.searchsorted(lb, xta, side="left") - 1
            cnt = np.maximum(last - first + 1, 0)
            A = np.repeat(ids, cnt)
            kk = np.arange(cnt.sum()) - np.repeat(np.cumsum(cnt) - cnt, cnt)
            Bl = np.repeat(first, cnt) + kk
            B = idb[Bl]
            lo = np.maximum(L[A], L[B]); hi = np.minimum(XT[A], XB[B])
            ok = (hi - lo) >= 0.05 * h
            A, B = A[ok], B[ok]
            left_b = L[B] >= L[A]               # left end of the overlap
            ci.append(np.where(left_b, B, A)); ck.append(np.where(left_b, 0, 3))
            cj.append(np.where(left_b, A, B))
            c2.append(np.where(left_b, 2, 0)); c3.append(np.where(left_b, 3, 1))
            right_b = XB[B] <= XT[A]            # right end of the overlap
            ci.append(np.where(right_b, B, A)); ck.append(np.where(right_b, 1, 2))
            cj.append(np.where(right_b, A, B))
            c2.append(np.where(right_b, 2, 0)); c3.append(np.where(right_b, 3, 1))
    ci = np.concatenate(ci); ck = np.concatenate(ck); cj = np.concatenate(cj)
    c2 = np.concatenate(c2); c3 = np.concatenate(c3)
    nc = ci.size
    assert ((c2 + 1) % 4 == c3).all()           # every contact edge runs to the next CCW vertex

    P1 = V[ci, ck]; P2 = V[cj, c2]; P3 = V[cj, c3]
    d = P3 - P2
    Le = np.linalg.norm(d, axis=1)
    t = d / Le[:, None]
    nrm = np.stack([t[:, 1], -t[:, 0]], axis=1)            # outward normal of a CCW edge
    tau = np.clip(((P1 - P2) * t).sum(axis=1) / Le, 0.0, 1.0)

    def ev(vec):
        return _t_transpose_times(P1[:, 0] - cx[ci], P1[:, 1] - cy[ci], vec[:, 0], vec[:, 1])

    def gv(vec):
        g2 = _t_transpose_times(P2[:, 0] - cx[cj], P2[:, 1] - cy[cj], vec[:, 0], vec[:, 1])
        g3 = _t_transpose_times(P3[:, 0] - cx[cj], P3[:, 1] - cy[cj], vec[:, 0], vec[:, 1])
        return -((1.0 - tau)[:, None] * g2 + tau[:, None] * g3)

    e_n, g_n = ev(nrm), gv(nrm)
    e_s, g_s = ev(t), gv(t)
    E_ref = 1.0
    pn0 = cfg.penalty * E_ref
    p_n = pn0 * (1.0 + rng.uniform(-0.2, 0.2, size=nc))
    locked = rng.random(nc) < cfg.lock_prob

    bi = np.concatenate([ci, ci[locked]]).astype(np.int32)
    bj = np.concatenate([cj, cj[locked]]).astype(np.int32)
    pen = np.concatenate([p_n, 0.4 * p_n[locked]])
    e = np.concatenate([e_n, e_s[locked]])
    g = np.concatenate([g_n, g_s[locked]])
    sp = rng.permutation(bi.size)              # contact detection emits springs in no order
    bi, bj, pen, e, g = bi[sp], bj[sp], pen[sp], np.ascontiguousarray(e[sp]), np.ascontiguousarray(g[sp])

    # ---------------- diagonal terms: elastic + inertia + fixed points
    band = np.minimum((course * len(MATERIAL_E)) // max(len(counts), 1), len(MATERIAL_E) - 1)
    Eb = np.asarray(MATERIAL_E)[band]
    kd = np.zeros((n, 6, 6))
    el = np.array([[1.0, NU, 0.0], [NU, 1.0, 0.0], [0.0, 0.0, 0.5 * (1.0 - NU)]]) / (1.0 - NU * NU)
    kd[:, 3:6, 3:6] += (area * Eb)[:, None, None] * el
    c_in = pn0 / (cfg.penalty_ratio * area.mean())
    kd += c_in * _inertia_integral(V, cx, cy)
    base = np.nonzero(course == 0)[0]
    pf = cfg.fixed_ratio * pn0
    for k in (0, 1):
        Tm = _t_matrix(V[base, k, 0] - cx[base], V[base, k, 1] - cy[base])   # [b,2,6]
        kd[base] += pf * np.einsum("bai,baj->bij", Tm, Tm)
    kd = 0.5 * (kd + np.transpose(kd, (0, 2, 1)))

    # ---------------- load: gravity on v0 plus a seeded perturbation on all six DOFs
    F = np.zeros((n, 6))
    F[:, 1] = -area
    F += 0.1 * area.mean() * rng.standard_normal((n, 6))
    F = F.reshape(-1)

    cent = np.stack([cx, cy], axis=1)
    cbi, cbj = ci, cj
    if cfg.shuffle:
        perm = rng.permutation(n)               # old id b -> new id perm[b]
        inv = np.empty_like(perm); inv[perm] = np.arange(n)
        kd = kd[inv]; course = course[inv]
        F = F.reshape(n, 6)[inv].reshape(-1)
        bi = perm[bi].astype(np.int32); bj = perm[bj].astype(np.int32)
        V = V[inv]; cent = cent[inv]
        cbi, cbj = perm[ci], perm[cj]
    contacts = {"i": cbi.astype(np.int32), "v": (4 * cbi + ck).astype(np.int32), "j": cbj.astype(np.int32),
                "e": (4 * cbj + c2).astype(np.int32), "tau": tau}

    return SlopeProblem(cfg=cfg, n=n, kdiag=np.ascontiguousarray(kd), bi=bi, bj=bj,
                        pen=pen, e=e, g=g, F=np.ascontiguousarray(F),
                        course=course.astype(np.int32), n_contacts=int(nc),
                        verts=np.ascontiguousarray(V), centroid=np.ascontiguousarray(cent), contacts=contacts)


def random_vector(n_blocks: int, seed: int) -> np.ndarray:
    """SpMV input x ~ U(-1, 1) of length 6n."""
    return np.random.default_rng(seed).uniform(-1.0, 1.0, size=6 * n_blocks)


def warm_start(d_ref: np.ndarray, seed: int, rel: float = 1e-3) -> np.ndarray:
    """Warm start d0 = d_ref * (1 + rel * N(0,1)) (ambiguity Z5)."""
    r = np.random.default_rng(seed).standard_normal(d_ref.shape)
    return d_ref * (1.0 + rel * r)


def case1_like(seed: int = 1046, n_blocks: int = 4361, n_offdiag: int = 18731):
    """A matrix input with the block counts of the paper's case 1 (4361 diagonal and 18731
    upper off-diagonal sub-matrices, u = 4.3, denser than a brick wall's u ~ 3): the jittered slope
    truncated to its first n_blocks blocks (springs between kept blocks only), plus one extra random
    spring (random e, g of the slope's scale, the slope's normal penalty) on distinct new block pairs
    (i, j), 2 <= j - i <= 3 * course length, drawn until there are exactly n_offdiag coupled pairs.
    Input generation only; returns (n, kdiag, bi, bj, pen, e, g, F)."""
    P = make_slope(preset(int(n_blocks * 1.05), seed=seed))
    assert P.n >= n_blocks
    keep = (P.bi < n_blocks) & (P.bj < n_blocks)
    bi, bj = P.bi[keep].astype(np.int64), P.bj[keep].astype(np.int64)
    pen, e, g = P.pen[keep], P.e[keep], P.g[keep]
    pairs = set(zip(np.minimum(bi, bj).tolist(), np.maximum(bi, bj).tolist()))
    assert len(pairs) <= n_offdiag
    rng = np.random.default_rng(seed + 1)
    L = int(np.bincount(P.course[:n_blocks]).max())
    scale_e, scale_g = float(np.abs(e).mean()), float(np.abs(g).mean())
    new_i, new_j = [], []
    while len(pairs) < n_offdiag:
        i = int(rng.integers(0, n_blocks - 2))
        j = i + int(rng.integers(2, 3 * L + 1))
        if j >= n_blocks or (i, j) in pairs:
            continue
        pairs.add((i, j))
        new_i.append(i)
        new_j.append(j)
    k = len(new_i)
    bi = np.concatenate([bi, new_i]).astype(np.int32)
    bj = np.concatenate([bj, new_j]).astype(np.int32)
    pen = np.concatenate([pen, np.full(k, float(P.pen.max()) / 1.2)])
    e = np.ascontiguousarray(np.concatenate([e, rng.normal(0.0, scale_e, (k, 6))]))
    g = np.ascontiguousarray(np.concatenate([g, rng.normal(0.0, scale_g, (k, 6))]))
    F = np.ascontiguousarray(P.F[:6 * n_blocks])
    return n_blocks, np.ascontiguousarray(P.kdiag[:n_blocks]), bi, bj, pen, e, g, F
