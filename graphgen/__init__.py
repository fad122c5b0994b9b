"""Seeded synthetic graph inputs shared by the oracle and the CUDA path.

Input plumbing only: this module holds none of the method's arithmetic (no
modularity, gains or community logic).  Every random draw is a pure function of
(seed, stream, index) (counter-based splitmix64, see graphgen.c), so graphs are
identical across runs and thread counts.

Configs follow BASELINE.json ``configs`` and the recipe in SURVEY.md §8(d)
(restated in DESIGN.md "Input recipe").  All level-0 graphs are symmetric,
unit-weight, self-loop free and duplicate free; vertex ids are randomly
permuted.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libgraphgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"graphgen: {path} missing - run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(path)
        i64, u64, dbl, p = ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p
        lib.gg_build_csr.restype = i64
        lib.gg_build_csr.argtypes = [i64, i64, p, p, p, ctypes.c_int, ctypes.c_int, p, p, p]
        lib.gg_rmat.restype = i64
        lib.gg_rmat.argtypes = [ctypes.c_int, i64, dbl, dbl, dbl, u64, i64, p, p]
        lib.gg_lfr.restype = i64
        lib.gg_lfr.argtypes = [i64, dbl, i64, dbl, dbl, i64, i64, dbl, u64, p, p, p, p]
        lib.gg_lfr_ex.restype = i64
        lib.gg_lfr_ex.argtypes = [i64, dbl, i64, dbl, dbl, i64, i64, dbl, u64, ctypes.c_int, dbl, ctypes.c_int,
                                  p, p, p, p]
        lib.gg_lfr_csr.restype = i64
        lib.gg_lfr_csr.argtypes = [i64, dbl, i64, dbl, dbl, i64, i64, dbl, u64, ctypes.c_int, p,
                                   ctypes.POINTER(ctypes.c_void_p), p, p, p]
        lib.gg_free.restype = None
        lib.gg_free.argtypes = [p]
        lib.gg_random_permutation.restype = None
        lib.gg_random_permutation.argtypes = [i64, u64, u64, p]
        lib.gg_rng_u64.restype = u64
        lib.gg_rng_u64.argtypes = [u64, u64, u64]
        _LIB = lib
    return _LIB


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


@dataclass
class CSR:
    """Symmetric CSR: row_ptr int64[n+1], col int32[nnz], w int64[nnz] or None (all 1)."""

    n: int
    row_ptr: np.ndarray
    col: np.ndarray
    w: np.ndarray | None = None
    name: str = ""
    truth: np.ndarray | None = None
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr)

    def weights(self) -> np.ndarray:
        return np.ones(self.nnz, dtype=np.int64) if self.w is None else self.w


def build_csr(n: int, src, dst, w=None, keep_self_loops: bool = False, merge_dups: bool = True,
              name: str = "") -> CSR:
    """Undirected edge list -> symmetric CSR (rows sorted, duplicates merged: weights summed when
    `w` is given, dropped (unit weight) when it is not).

    A pair (u, v), u != v, yields entries (u, v) and (v, u); a self loop (v, v, w)
    yields one entry (v, v, w) when kept (the library's convention: stored once,
    counted once in d(v), see include/gala.h).
    """
    src = np.ascontiguousarray(src, dtype=np.int64)
    dst = np.ascontiguousarray(dst, dtype=np.int64)
    m = int(src.shape[0])
    wa = None if w is None else np.ascontiguousarray(w, dtype=np.int64)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    col = np.zeros(max(2 * m, 1), dtype=np.int32)
    wout = np.zeros(max(2 * m, 1), dtype=np.int64)
    nnz = _lib().gg_build_csr(n, m, _ptr(src), _ptr(dst), _ptr(wa), int(keep_self_loops),
                              int(merge_dups), _ptr(row_ptr), _ptr(col), _ptr(wout))
    if nnz < 0:
        raise ValueError("edge endpoint out of range")
    col = col[:nnz].copy()
    if w is None:
        # unweighted input: duplicates are dropped (simple graph, unit weights)
        return CSR(n=n, row_ptr=row_ptr, col=col, w=None, name=name)
    wout = wout[:nnz].copy()
    return CSR(n=n, row_ptr=row_ptr, col=col, w=wout, name=name)


def random_permutation(n: int, seed: int, stream: int = 0) -> np.ndarray:
    perm = np.zeros(n, dtype=np.int64)
    _lib().gg_random_permutation(n, seed, stream, _ptr(perm))
    return perm


# --------------------------------------------------------------------------
# Zachary karate club (Zachary 1977, "An information flow model for conflict
# and fission in small groups", J. Anthropol. Res. 33:452-473), 34 vertices,
# 78 undirected edges, 0-indexed as in networkx.karate_club_graph().
# --------------------------------------------------------------------------
KARATE_ADJ = {
    0: [1, 2, 3, 4, 5, 6, 7, 8, 10, 11, 12, 13, 17, 19, 21, 31],
    1: [2, 3, 7, 13, 17, 19, 21, 30],
    2: [3, 7, 8, 9, 13, 27, 28, 32],
    3: [7, 12, 13],
    4: [6, 10],
    5: [6, 10, 16],
    6: [16],
    8: [30, 32, 33],
    9: [33],
    13: [33],
    14: [32, 33],
    15: [32, 33],
    18: [32, 33],
    19: [33],
    20: [32, 33],
    22: [32, 33],
    23: [25, 27, 29, 32, 33],
    24: [25, 27, 31],
    25: [31],
    26: [29, 33],
    27: [33],
    28: [31, 33],
    29: [32, 33],
    30: [32, 33],
    31: [32, 33],
    32: [33],
}


def karate_edges():
    src, dst = [], []
    for u, vs in KARATE_ADJ.items():
        for v in vs:
            src.append(u)
            dst.append(v)
    return 34, np.array(src, dtype=np.int64), np.array(dst, dtype=np.int64)


def karate() -> CSR:
    n, s, d = karate_edges()
    return build_csr(n, s, d, name="karate")


def rmat(scale: int, n: int, m_target: int, a=0.48, b=0.20, c=0.20, seed=2, name="rmat") -> CSR:
    """R-MAT with quadrant probabilities (a, b, c, 1-a-b-c), m_target distinct undirected edges."""
    src = np.zeros(m_target, dtype=np.int64)
    dst = np.zeros(m_target, dtype=np.int64)
    m = _lib().gg_rmat(scale, n, a, b, c, seed, m_target, _ptr(src), _ptr(dst))
    g = build_csr(n, src[:m], dst[:m], name=name)
    g.meta.update(dict(generator="rmat", scale=scale, a=a, b=b, c=c, seed=seed, m_target=m_target))
    return g


def lfr(n: int, avg_k: float, kmax: int, mu: float, tau1=2.5, tau2=1.5, cmin=50, cmax=2000,
        seed=1, name="lfr", fit_frac: bool = False, alpha: float = 1.0, rewire: bool = False) -> CSR:
    """LFR-style planted partition (see graphgen.c gg_lfr_ex for the steps).

    fit_frac: fit the degree law's mean to avg_k exactly (fractional weight on k_min) instead of
    the nearest integer k_min.  alpha: a vertex's internal degree is at most alpha * (size - 1) of
    its community (the excess becomes external stubs); alpha = 1 is the classic LFR bound.
    rewire: self pairs, duplicates and external pairs inside one community are repaired by
    degree-preserving double-edge swaps instead of being dropped."""
    lib = _lib()
    ub = lib.gg_lfr_ex(n, avg_k, kmax, tau1, tau2, cmin, cmax, mu, seed, int(fit_frac), alpha, int(rewire),
                       None, None, None, None)
    src = np.zeros(ub, dtype=np.int64)
    dst = np.zeros(ub, dtype=np.int64)
    truth = np.zeros(n, dtype=np.int64)
    kmin = ctypes.c_int64(0)
    m = lib.gg_lfr_ex(n, avg_k, kmax, tau1, tau2, cmin, cmax, mu, seed, int(fit_frac), alpha, int(rewire),
                      _ptr(src), _ptr(dst), _ptr(truth), ctypes.byref(kmin))
    g = build_csr(n, src[:m], dst[:m], name=name)
    g.truth = truth
    g.meta.update(dict(generator="lfr", avg_k=avg_k, kmax=kmax, kmin=int(kmin.value), mu=mu,
                       tau1=tau1, tau2=tau2, cmin=cmin, cmax=cmax, seed=seed, fit_frac=fit_frac,
                       alpha=alpha, rewire=rewire))
    return g


def lfr_csr(n: int, avg_k: float, kmax: int, mu: float, tau1=2.5, tau2=1.5, cmin=50, cmax=2000, seed=1,
            name="lfr", fit_frac: bool = False) -> CSR:
    """Memory-lean LFR-style graph built straight into CSR (graphgen.c gg_lfr_csr): the plan of
    lfr() (degrees, community sizes, placement, internal wiring), external stubs paired through a
    counter-based random bijection instead of a sort, self pairs / duplicates / same-community
    external pairs dropped.  For the Friendster shape (1.8B edges), whose edge list does not fit
    the host twice over.  The column array is owned by the returned CSR (freed with it)."""
    import weakref
    lib = _lib()
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    truth = np.zeros(n, dtype=np.int64)
    colp = ctypes.c_void_p()
    kmin = ctypes.c_int64(0)
    stats = np.zeros(3, dtype=np.int64)
    nnz = lib.gg_lfr_csr(n, avg_k, kmax, tau1, tau2, cmin, cmax, mu, seed, int(fit_frac), _ptr(row_ptr), ctypes.byref(colp),
                         _ptr(truth), ctypes.byref(kmin), _ptr(stats))
    col = np.ctypeslib.as_array(ctypes.cast(colp, ctypes.POINTER(ctypes.c_int32)), shape=(max(nnz, 1),))[:nnz]
    weakref.finalize(col.base, lib.gg_free, colp.value)
    g = CSR(n=n, row_ptr=row_ptr, col=col, w=None, name=name, truth=truth)
    g.meta.update(dict(generator="lfr_csr", avg_k=avg_k, kmax=kmax, kmin=int(kmin.value), mu=mu, tau1=tau1,
                       tau2=tau2, cmin=cmin, cmax=cmax, seed=seed, fit_frac=fit_frac, internal_edges=int(stats[0]),
                       external_pairs=int(stats[1]), dropped=int(stats[2])))
    return g


def random_graph(n: int, m: int, seed: int, max_w: int = 1, self_loops: int = 0) -> CSR:
    """Small seeded random multigraph for tests (numpy Generator; merges duplicates).

    max_w > 1 draws integer weights in [1, max_w]; self_loops adds that many
    (v, v, w) entries.
    """
    rng = np.random.default_rng(seed)
    s = rng.integers(0, n, size=m)
    d = rng.integers(0, n, size=m)
    keep = s != d
    s, d = s[keep], d[keep]
    w = rng.integers(1, max_w + 1, size=s.shape[0]) if max_w > 1 else None
    if self_loops:
        ls = rng.integers(0, n, size=self_loops)
        lw = rng.integers(1, max(max_w, 2) + 1, size=self_loops)
        w0 = w if w is not None else np.ones(s.shape[0], dtype=np.int64)
        s = np.concatenate([s, ls])
        d = np.concatenate([d, ls])
        w = np.concatenate([w0, lw])
    return build_csr(n, s, d, w, keep_self_loops=bool(self_loops), name=f"rand{n}_{m}_{seed}")


def ring_of_cliques(r: int, s: int) -> CSR:
    """r cliques K_s joined in a ring by single edges (clique i vertex 0 -- clique i+1 vertex 1)."""
    src, dst = [], []
    for i in range(r):
        base = i * s
        for a in range(s):
            for b in range(a + 1, s):
                src.append(base + a)
                dst.append(base + b)
        if r > 1 and not (r == 2 and i == 1):
            src.append(base)
            dst.append(((i + 1) % r) * s + 1)
    return build_csr(r * s, np.array(src), np.array(dst), name=f"ring{r}xK{s}")


# --------------------------------------------------------------------------
# BASELINE.json configs (SURVEY.md §8(d) recipe)
# --------------------------------------------------------------------------
CONFIGS = {
    "karate": dict(desc="Zachary karate club, 34 V / 78 E (embedded edge list)"),
    "lfr1m": dict(desc="LFR planted partition, n=1e6, <k>=40, kmax=1000, tau1=2.5, tau2=1.5, "
                       "c in [50,2000], mu=0.3, seed 1"),
    "rmat_lj": dict(desc="R-MAT scale 23 (0.48,0.20,0.20,0.12), n=4,847,571, 69.0M undirected edges, seed 2"),
    "orkut": dict(desc="LFR-style n=3,072,441, <k>=76.3 (m=117.2M), kmax=33,313, tau1=2.3, c in [50,50000], "
                       "mu=0.35, internal degree <= (size-1)/2, rewired to a simple graph, seed 3"),
    "friendster": dict(desc="LFR-style n=65,608,366, realised <k>=55.06 (1.806B edges), kmax=5,214, tau1=2.5, mu=0.37, "
                            "seed 4; memory-lean "
                            "generator straight to CSR (gg_lfr_csr: external stubs paired by a counter-based "
                            "bijection; ~30 GB host, minutes on 16 cores)"),
    # the Friendster shape at 1/4 of its vertices (same degree law / mixing): the largest FR-shaped
    # graph one GPU-box host generates comfortably; C + Sigma_tot (197 MB) exceed the 126 MB L2
    "friendster_q": dict(desc="LFR-style n=16,402,092, <k>=55.06, kmax=5,214, tau1=2.5, mu=0.37, seed 4"),
    # scaled-down shapes for tests (same recipe, smaller n)
    "lfr_small": dict(desc="LFR n=20,000, <k>=20, kmax=200, mu=0.3, seed 11"),
    "lfr_mid": dict(desc="LFR n=200,000, <k>=40, kmax=1000, mu=0.3, seed 12"),
    "rmat_small": dict(desc="R-MAT scale 15, n=30,000, 300k edges, seed 13"),
    # Table 4-style NMI graphs (LFR, 100,000 vertices, 0.65M / 1.44M / 1.44M edges;
    # the paper does not give their mixing, so three mixing levels are used)
    "lfr100k_1": dict(desc="LFR n=100,000, <k>=13, kmax=100, mu=0.5, seed 21"),
    "lfr100k_2": dict(desc="LFR n=100,000, <k>=29, kmax=300, mu=0.1, seed 22"),
    "lfr100k_3": dict(desc="LFR n=100,000, <k>=29, kmax=300, mu=0.45, seed 23"),
}


def make(name: str) -> CSR:
    if name == "karate":
        return karate()
    if name == "lfr1m":
        return lfr(1_000_000, 40.0, 1000, 0.3, seed=1, name=name)
    if name == "rmat_lj":
        return rmat(23, 4_847_571, 69_000_000, seed=2, name=name)
    if name == "orkut":
        # tau1 = 2.3 (not the survey's 2.0): a tau1 = 2.0 law truncated at 33,313 puts ~16 % of all
        # stubs on ~2,100 vertices of degree > 10^4, more hub-hub pairs than a simple graph holds, so
        # it realises only 102.7M edges with max degree 23k (measured).  avg_k 76.68 = 76.3 scaled by
        # the 0.5 % the rewiring still drops; realised: 117.2M edges, max degree 33.1k
        return lfr(3_072_441, 76.68, 33_313, 0.35, tau1=2.3, cmin=50, cmax=50000, seed=3, name=name,
                   fit_frac=True, alpha=0.5, rewire=True)
    if name == "friendster":
        # avg_k 63.85 with the exact-mean law: the configuration-model wiring drops ~13.8 % of the
        # pairs (duplicates inside small dense communities, same-community external pairs), so the
        # law's mean is raised until the REALISED mean degree is FR's 55.06 (1.806B edges;
        # calibrated at n = 2M: 63 -> 54.35, 64 -> 55.18; the drop fraction does not depend on n)
        return lfr_csr(65_608_366, 63.85, 5_214, 0.37, seed=4, name=name, fit_frac=True)
    if name == "friendster_q":
        return lfr(16_402_092, 55.06, 5_214, 0.37, seed=4, name=name)
    if name == "lfr_small":
        return lfr(20_000, 20.0, 200, 0.3, cmin=20, cmax=500, seed=11, name=name)
    if name == "lfr_mid":
        return lfr(200_000, 40.0, 1000, 0.3, seed=12, name=name)
    if name == "rmat_small":
        return rmat(15, 30_000, 300_000, seed=13, name=name)
    if name == "lfr100k_1":
        return lfr(100_000, 13.0, 100, 0.5, cmin=20, cmax=1000, seed=21, name=name)
    if name == "lfr100k_2":
        return lfr(100_000, 29.0, 300, 0.1, cmin=20, cmax=1000, seed=22, name=name)
    if name == "lfr100k_3":
        return lfr(100_000, 29.0, 300, 0.45, cmin=20, cmax=1000, seed=23, name=name)
    raise KeyError(name)
