"""CPU oracle of GALA's Louvain (ctypes binding of oracle/gala_oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this module.  The product
path (paper_conf_ppopp_wangllwm00z25_b200) never imports it and shares no
code with it.  See gala_oracle.c's header for what each function follows in
the paper (Eq. 1, Eq. 2, Alg. 1, Eq. 6/7, §2.2 phase 2).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"oracle: {path} missing - run `make`")
        lib = ctypes.CDLL(path)
        i64, i32, dbl, p = ctypes.c_int64, ctypes.c_int32, ctypes.c_double, ctypes.c_void_p
        lib.oracle_louvain.restype = p
        lib.oracle_louvain.argtypes = [i64, p, p, p, dbl, dbl, i32, i32, ctypes.c_int, ctypes.c_int,
                                       ctypes.c_int]
        lib.oracle_status.restype = ctypes.c_int
        lib.oracle_status.argtypes = [p]
        lib.oracle_num_communities.restype = i64
        lib.oracle_num_communities.argtypes = [p]
        lib.oracle_labels.restype = None
        lib.oracle_labels.argtypes = [p, p]
        lib.oracle_summary.restype = None
        lib.oracle_summary.argtypes = [p, p]
        lib.oracle_modularity.restype = dbl
        lib.oracle_modularity.argtypes = [p]
        lib.oracle_record.restype = None
        lib.oracle_record.argtypes = [p, i64, p]
        lib.oracle_record_labels.restype = ctypes.c_int
        lib.oracle_record_labels.argtypes = [p, i64, p]
        lib.oracle_record_pruned.restype = ctypes.c_int
        lib.oracle_record_pruned.argtypes = [p, i64, p]
        lib.oracle_level.restype = None
        lib.oracle_level.argtypes = [p, i64, p]
        lib.oracle_free.restype = None
        lib.oracle_free.argtypes = [p]
        lib.oracle_partition_numerator.restype = ctypes.c_int
        lib.oracle_partition_numerator.argtypes = [i64, p, p, p, p, dbl, p]
        lib.oracle_move_gain.restype = None
        lib.oracle_move_gain.argtypes = [i64, p, p, p, p, dbl, i64, i32, p]
        lib.oracle_gamma_pq.restype = None
        lib.oracle_gamma_pq.argtypes = [dbl, p, p]
        _LIB = lib
    return _LIB


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _i128(hi, lo) -> int:
    return (int(hi) << 64) | (int(lo) & 0xFFFFFFFFFFFFFFFF)


def _csr_arrays(g):
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(g.col, dtype=np.int32)
    w = None if g.w is None else np.ascontiguousarray(g.w, dtype=np.int64)
    return rp, col, w


@dataclass
class IterRecord:
    level: int
    iter: int
    n_level: int
    n_active: int
    n_pruned: int
    n_moved: int
    n_fn: int
    N: int
    labels: np.ndarray | None
    n_fp: int = 0
    pruned: np.ndarray | None = None   # trace >= 3: per-vertex inactive flags (bool)


@dataclass
class LevelRecord:
    n: int
    nnz: int
    iters: int
    N_start: int
    N_end: int


@dataclass
class OracleResult:
    status: int
    labels: np.ndarray
    k: int
    W: int
    p: int
    q: int
    N: int
    Q: float
    records: list
    levels: list


def gamma_pq(gamma: float):
    p = ctypes.c_int64()
    q = ctypes.c_int64()
    _lib().oracle_gamma_pq(gamma, ctypes.byref(p), ctypes.byref(q))
    return p.value, q.value


PRUNE_NONE, PRUNE_MG, PRUNE_SM, PRUNE_RM, PRUNE_MG_RM = 0, 1, 2, 3, 4


def louvain(g, gamma: float = 1.0, tol: float = 1e-6, max_levels: int = 0, max_iters: int = 0,
            prune: int = 0, check: bool = False, trace: int = 1) -> OracleResult:
    """Run the oracle's multi-level BSP Louvain on CSR `g` (graphgen.CSR-like).

    prune: 0/False none, 1/True MG (Eq. 6/7), 2 SM, 3 RM, 4 MG+RM (§3.2-3.3; DESIGN.md c20/c21).
    check: also evaluate pruned vertices -> per-iteration false negatives (n_fn) and, for the
    active set, false positives (n_fp) in the records.
    trace: 1 records, 2 + label snapshots, 3 + per-vertex inactive flags (IterRecord.pruned)."""
    lib = _lib()
    rp, col, w = _csr_arrays(g)
    h = lib.oracle_louvain(g.n, _ptr(rp), _ptr(col), _ptr(w), gamma, tol, max_levels, max_iters,
                           int(prune), int(check), int(trace))
    try:
        st = lib.oracle_status(h)
        summ = np.zeros(7, dtype=np.int64)
        lib.oracle_summary(h, _ptr(summ))
        labels = np.zeros(g.n, dtype=np.int32)
        lib.oracle_labels(h, _ptr(labels))
        recs = []
        buf = np.zeros(10, dtype=np.int64)
        for i in range(int(summ[6])):
            lib.oracle_record(h, i, _ptr(buf))
            lab = None
            pf = None
            if trace >= 2:
                lab = np.zeros(int(buf[2]), dtype=np.int32)
                lib.oracle_record_labels(h, i, _ptr(lab))
            if trace >= 3:
                pf = np.zeros(int(buf[2]), dtype=np.uint8)
                lib.oracle_record_pruned(h, i, _ptr(pf))
                pf = pf.astype(bool)
            recs.append(IterRecord(int(buf[0]), int(buf[1]), int(buf[2]), int(buf[3]), int(buf[4]),
                                   int(buf[5]), int(buf[6]), _i128(buf[7], buf[8]), lab, int(buf[9]), pf))
        levs = []
        lb = np.zeros(7, dtype=np.int64)
        for i in range(int(summ[5])):
            lib.oracle_level(h, i, _ptr(lb))
            levs.append(LevelRecord(int(lb[0]), int(lb[1]), int(lb[2]), _i128(lb[3], lb[4]),
                                    _i128(lb[5], lb[6])))
        return OracleResult(status=st, labels=labels, k=int(lib.oracle_num_communities(h)),
                            W=int(summ[0]), p=int(summ[1]), q=int(summ[2]),
                            N=_i128(summ[3], summ[4]), Q=float(lib.oracle_modularity(h)),
                            records=recs, levels=levs)
    finally:
        lib.oracle_free(h)


def partition_numerator(g, labels, gamma: float = 1.0):
    """(W, N) for an arbitrary partition: N = q W sum D_C - p sum D_V^2 (Eq. 1 x q W^2)."""
    rp, col, w = _csr_arrays(g)
    lab = np.ascontiguousarray(labels, dtype=np.int32)
    out = np.zeros(3, dtype=np.int64)
    if _lib().oracle_partition_numerator(g.n, _ptr(rp), _ptr(col), _ptr(w), _ptr(lab), gamma,
                                         _ptr(out)):
        raise ValueError("invalid labels")
    return int(out[0]), _i128(out[1], out[2])


def modularity(g, labels, gamma: float = 1.0) -> float:
    W, N = partition_numerator(g, labels, gamma)
    p, q = gamma_pq(gamma)
    return 0.0 if W == 0 else N / (q * W * W)


def move_gain2(g, labels, v: int, target: int, gamma: float = 1.0) -> int:
    """Closed form 2*(score(target) - stay) for moving v (Eq. 2, reading c1)."""
    rp, col, w = _csr_arrays(g)
    lab = np.ascontiguousarray(labels, dtype=np.int32)
    out = np.zeros(2, dtype=np.int64)
    _lib().oracle_move_gain(g.n, _ptr(rp), _ptr(col), _ptr(w), _ptr(lab), gamma, v, target, _ptr(out))
    return _i128(out[0], out[1])
