"""Statistics checks of the memory-lean LFR generator (graphgen.lfr_csr / gg_lfr_csr) that builds
the full Friendster shape: it is input plumbing shared by both sides ("parity unpinned",
statistics only), so these tests pin what the recipe promises -- a simple symmetric graph with
sorted, duplicate-free rows, the planted membership, the degree law's bounds, the mixing, and
determinism for any thread count -- at sizes that run in seconds."""
import hashlib
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import graphgen as gg  # noqa: E402


def _digest(g):
    return hashlib.sha1(g.row_ptr.tobytes() + np.asarray(g.col).tobytes() + g.truth.tobytes()).hexdigest()


def test_lean_lfr_is_simple_symmetric_and_sorted():
    g = gg.lfr_csr(60_000, 30.0, 600, 0.3, seed=7)
    n, rp, col = g.n, g.row_ptr, np.asarray(g.col)
    deg = np.diff(rp)
    row = np.repeat(np.arange(n, dtype=np.int64), deg)
    assert rp[0] == 0 and rp[-1] == g.nnz and (deg >= 0).all()
    assert ((col >= 0) & (col < n)).all()
    assert (col != row).all()                                   # no self loops
    key = row * n + col
    assert (np.diff(key) > 0).all()                             # rows sorted, no duplicates
    assert np.array_equal(np.sort(col.astype(np.int64) * n + row), key)   # symmetric
    assert deg.max() <= 600
    assert g.truth.shape == (n,) and g.truth.min() >= 0
    sizes = np.bincount(g.truth)
    assert sizes[sizes > 0].min() >= 20                         # remainders are spread (c_min = 50)
    mu = (g.truth[row] != g.truth[col]).mean()
    assert 0.25 < mu < 0.40                                     # target 0.3 (drops shift it a little)
    m = g.meta
    assert m["internal_edges"] + m["external_pairs"] - m["dropped"] == g.nnz // 2


def test_lean_lfr_exact_mean_fit_and_seed():
    a = gg.lfr_csr(40_000, 25.0, 400, 0.35, seed=3, fit_frac=True)
    b = gg.lfr_csr(40_000, 25.0, 400, 0.35, seed=3, fit_frac=True)
    c = gg.lfr_csr(40_000, 25.0, 400, 0.35, seed=4, fit_frac=True)
    assert _digest(a) == _digest(b) and _digest(a) != _digest(c)
    # the exact-mean law has mean 25 before the configuration-model drops
    stubs = 2 * (a.meta["internal_edges"] + a.meta["external_pairs"])
    assert abs(stubs / a.n - 25.0) < 0.5


def test_lean_lfr_independent_of_thread_count():
    code = ("import sys; sys.path.insert(0, %r); import graphgen as gg, hashlib, numpy as np; "
            "g = gg.lfr_csr(30_000, 20.0, 300, 0.3, seed=9); "
            "print(hashlib.sha1(g.row_ptr.tobytes() + np.asarray(g.col).tobytes() + g.truth.tobytes()).hexdigest())"
            % ROOT)
    out = []
    for t in ("1", "4"):
        env = dict(os.environ, OMP_NUM_THREADS=t)
        out.append(subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env,
                                  check=True).stdout.strip())
    assert out[0] == out[1]
