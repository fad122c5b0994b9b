"""NMI of two partitions (Table 4; definition of ref. [52], Strehl & Ghosh
2002, "Cluster ensembles", JMLR 3:583-617, Eq. 2 there): the mutual information of the two
label variables normalised by the geometric mean of their entropies,

    NMI(X, Y) = I(X; Y) / sqrt(H(X) H(Y)),
    I(X; Y)   = sum_{a,b} (n_ab / n) log( n n_ab / (n_a n_b) ),
    H(X)      = -sum_a (n_a / n) log(n_a / n),

with n_ab the contingency counts.  Convention for the degenerate case (one side has a single
cluster, H = 0): NMI = 1 if both sides are single-cluster, else 0 (no information shared).

TEST INFRASTRUCTURE ONLY (same rule as oracle/__init__.py): fp64, plain numpy, written from
the definition; pinned by tests/test_oracle_nmi.py (hand-computed example, identity, product
partitions, relabelling invariance, symmetry, scikit-learn's geometric NMI).
"""
from __future__ import annotations

import numpy as np


def nmi(x, y) -> float:
    x = np.asarray(x, dtype=np.int64).ravel()
    y = np.asarray(y, dtype=np.int64).ravel()
    if x.shape != y.shape:
        raise ValueError("nmi: partitions of different length")
    n = x.size
    if n == 0:
        return 1.0
    _, xi = np.unique(x, return_inverse=True)
    _, yi = np.unique(y, return_inverse=True)
    kx, ky = int(xi.max()) + 1, int(yi.max()) + 1
    na = np.bincount(xi, minlength=kx).astype(np.float64)
    nb = np.bincount(yi, minlength=ky).astype(np.float64)
    # contingency counts n_ab over the pairs that occur
    pair, nab = np.unique(xi * ky + yi, return_counts=True)
    a, b = pair // ky, pair % ky
    nab = nab.astype(np.float64)
    I = float(np.sum(nab / n * np.log(n * nab / (na[a] * nb[b]))))
    hx = float(-np.sum(na / n * np.log(na / n)))
    hy = float(-np.sum(nb / n * np.log(nb / n)))
    if hx == 0.0 or hy == 0.0:
        return 1.0 if hx == hy else 0.0
    return I / np.sqrt(hx * hy)
