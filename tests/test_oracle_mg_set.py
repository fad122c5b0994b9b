"""Pin of the MG inactive SET (Eq. 6/7) — not just its soundness.

For every iteration of every level the state at the start of the iteration is rebuilt here in
numpy from nothing but the level-0 CSR and the oracle's label trace:
  * the level graph: level-0 entries (u, v, w) aggregated by (map[u], map[v]) — a stored self
    loop counts once in d(v); the diagonal of a super vertex is the weight of every entry inside
    it (reading c10);
  * d(v) = row sum, s(v) = diagonal, d'(v) = d_{C[v]}(v) = weight to C[v] without the diagonal
    (reading c2), Sigma_tot(c) = D_V(c) = sum of d over the members;
  * min_C D_V(C) over the non-empty communities (reading c3);
  * Eq. 6 exactly as printed, 2 d' - d + (min D_V - D_V(C[v])) * gamma * d / 2|E| >= 0, in
    exact rational arithmetic (gamma = p/q, reading c11), for every v with d(v) > 0;
  * the next level's vertex ids in min-member order (reading c9).
The recomputed set must equal the oracle's per-vertex inactive flags (trace=3) in every
iteration.  Two plausible wrong readings — min over ALL communities (empty ones included, c3)
and a conservative Eq. 6 (d instead of 2 d' - d, i.e. dropping d'), — must give a different
set somewhere on these graphs, so an oracle built on either would fail this test.

Also the survey-time independent karate trace: pruned counts [0, 3, 7] on
level 0, 34 -> 9 -> 4 communities, final N = 10154 (tests/golden/karate_trace.json).
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import graphgen as gg
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "karate_trace.json")


def _entries(g):
    rows = np.repeat(np.arange(g.n, dtype=np.int64), np.diff(g.row_ptr))
    return rows, g.col.astype(np.int64), g.weights().astype(np.int64)


def _level_quantities(rows, cols, w, vmap, n_level):
    """d, s per level vertex from the level-0 entries mapped through vmap (level-0 -> level)."""
    r, c = vmap[rows], vmap[cols]
    d = np.zeros(n_level, dtype=np.int64)
    np.add.at(d, r, w)
    s = np.zeros(n_level, dtype=np.int64)
    diag = r == c
    np.add.at(s, r[diag], w[diag])
    return r, c, d, s


def _inactive(r, c, w, d, s, C, gamma_pq, W, rule="paper"):
    """Eq. 6/7 inactive flags for the level state (C = community of every level vertex)."""
    p, q = gamma_pq
    n = d.shape[0]
    off = r != c
    same = off & (C[r] == C[c])
    dp = np.zeros(n, dtype=np.int64)
    np.add.at(dp, r[same], w[same])
    sig = np.zeros(n, dtype=np.int64)
    np.add.at(sig, C, d)
    if rule == "min_all":            # wrong reading of c3: empty communities included
        mins = int(sig.min())
    else:
        mins = int(sig[sig > 0].min())
    gamma = Fraction(p, q)
    out = np.zeros(n, dtype=bool)
    for v in range(n):
        dv = int(d[v])
        if dv == 0:
            continue
        own = 2 * int(dp[v]) - dv if rule != "no_dprime" else -dv
        lhs = own + (mins - int(sig[C[v]])) * gamma * Fraction(dv, W)
        out[v] = lhs >= 0
    return out


def _recount(g, res, gamma, rule="paper"):
    """Yield (level, iter, recomputed flags, oracle record) for every iteration of `res`."""
    rows, cols, w = _entries(g)
    W = int(w.sum())
    pq = oracle.gamma_pq(gamma)
    vmap = np.arange(g.n, dtype=np.int64)
    recs = res.records
    i = 0
    level = 0
    while i < len(recs):
        n_level = recs[i].n_level
        r, c, d, s = _level_quantities(rows, cols, w, vmap, n_level)
        C = np.arange(n_level, dtype=np.int64)
        while i < len(recs) and recs[i].level == level:
            yield level, recs[i].iter, _inactive(r, c, w, d, s, C, pq, W, rule), recs[i]
            C = recs[i].labels.astype(np.int64)
            i += 1
        # next level ids: communities in order of their smallest member (c9)
        first = np.full(n_level, np.iinfo(np.int64).max, dtype=np.int64)
        np.minimum.at(first, C, np.arange(n_level, dtype=np.int64))
        used = np.unique(C)
        order = used[np.argsort(first[used], kind="stable")]
        newid = np.full(n_level, -1, dtype=np.int64)
        newid[order] = np.arange(order.shape[0])
        vmap = newid[C[vmap]]
        level += 1


def _cases():
    out = [("karate", gg.karate(), 1.0), ("lfr_small", gg.make("lfr_small"), 1.0),
           ("rmat_small", gg.make("rmat_small"), 1.0)]
    for seed in range(3):
        for gamma in (0.5, 1.0, 2.0):
            out.append((f"rand{seed}_g{gamma}", gg.random_graph(150, 900, seed=7100 + seed, max_w=4, self_loops=5),
                        gamma))
    return out


CASES = _cases()


@pytest.mark.parametrize("ci", range(len(CASES)), ids=[c[0] for c in CASES])
def test_mg_inactive_set_equals_eq6_recount(ci):
    name, g, gamma = CASES[ci]
    res = oracle.louvain(g, gamma=gamma, prune=1, trace=3)
    assert res.status == 0
    n_iters = 0
    for level, it, flags, rec in _recount(g, res, gamma):
        assert rec.pruned is not None
        assert np.array_equal(flags, rec.pruned), f"{name} level {level} iter {it}"
        assert int(flags.sum()) == rec.n_pruned
        n_iters += 1
    assert n_iters == len(res.records)


def test_wrong_readings_are_detected():
    """The recount distinguishes the paper's reading from two plausible mistakes: on these
    graphs each wrong rule yields a different inactive set in some iteration, so an oracle that
    implemented it would fail test_mg_inactive_set_equals_eq6_recount."""
    differs = {"min_all": False, "no_dprime": False}
    for name, g, gamma in CASES[:6]:
        res = oracle.louvain(g, gamma=gamma, prune=1, trace=3)
        for rule in differs:
            if differs[rule]:
                continue
            for _, _, flags, rec in _recount(g, res, gamma, rule=rule):
                if not np.array_equal(flags, rec.pruned):
                    differs[rule] = True
                    break
    assert all(differs.values()), differs


def test_karate_survey_trace():
    """SURVEY.md §8(c) P8 (a survey-time independent re-implementation, not this oracle):
    level-0 pruned counts [0, 3, 7], 34 -> 9 -> 4 communities, final N = 10154 (Q = 0.417242)."""
    gold = json.load(open(GOLDEN))
    res = oracle.louvain(gg.karate(), prune=1, trace=2)
    lv0 = [r.n_pruned for r in res.records if r.level == 0]
    assert lv0 == gold["level0_pruned"]
    assert [lv.n for lv in res.levels] == gold["level_sizes"]
    assert res.k == gold["communities"]
    assert res.N == gold["N"]
    assert abs(res.Q - gold["Q_6dp"]) < 5e-7
