"""Oracle pins of the pruning strategies of §3.2-3.3: none, MG (Eq. 6/7),
SM (strict movement), RM (relaxed movement), MG+RM.

Pinned against the paper's lemmas and against the strategies' definitions re-derived here
from the oracle's label trace (readings c20/c21 in DESIGN.md):
  * Lemma 3 / Theorem 6: SM and MG have no false negatives and leave every label unchanged;
  * Lemma 4: RM can prune a vertex that would move (false negatives > 0, labels differ);
  * MG prunes only vertices that stay, so MG+RM makes exactly RM's moves (Table 3 lists
    "RM/MG+RM" as one column);
  * Eq. 3 bookkeeping: moved = active - false positives in every iteration;
  * iteration 1 of level 0: the SM and RM pruned counts equal those recomputed in Python from
    the iteration-0 moves, and MG+RM prunes the union of the MG and RM sets.
"""
import numpy as np
import pytest

import graphgen as gg
import oracle

NONE, MG, SM, RM, MGRM = 0, 1, 2, 3, 4


def graphs():
    out = [gg.karate(), gg.make("lfr_small")]
    for seed in range(4):
        out.append(gg.random_graph(200, 1200, seed=4000 + seed, max_w=3, self_loops=3))
    return out


@pytest.mark.parametrize("gi", range(6))
def test_lossless_strategies_keep_every_label(gi):
    g = graphs()[gi]
    base = oracle.louvain(g, prune=NONE, trace=2)
    for mode in (MG, SM):
        o = oracle.louvain(g, prune=mode, check=True, trace=2)
        assert o.status == 0
        assert np.array_equal(o.labels, base.labels)
        assert o.N == base.N
        assert len(o.records) == len(base.records)
        for x, y in zip(o.records, base.records):
            assert np.array_equal(x.labels, y.labels)
            assert x.n_moved == y.n_moved
            assert x.n_fn == 0                        # Lemma 3 / Theorem 6
            assert x.n_active + x.n_pruned == y.n_active


@pytest.mark.parametrize("gi", range(6))
def test_mg_rm_makes_exactly_the_rm_moves(gi):
    g = graphs()[gi]
    rm = oracle.louvain(g, prune=RM, check=True, trace=2)
    both = oracle.louvain(g, prune=MGRM, check=True, trace=2)
    assert np.array_equal(rm.labels, both.labels) and rm.N == both.N
    assert len(rm.records) == len(both.records)
    for x, y in zip(rm.records, both.records):
        assert np.array_equal(x.labels, y.labels)
        assert x.n_moved == y.n_moved and x.n_fn == y.n_fn
        assert y.n_pruned >= x.n_pruned               # MG only adds pruned vertices


@pytest.mark.parametrize("mode", [NONE, MG, SM, RM, MGRM])
def test_moved_equals_active_minus_false_positives(mode):
    for g in graphs()[:3]:
        o = oracle.louvain(g, prune=mode, check=True, trace=1)
        for r in o.records:
            assert r.n_moved == r.n_active - r.n_fp
            if mode in (NONE, MG, SM):
                assert r.n_fn == 0
        if mode == NONE:
            assert all(r.n_pruned == 0 for r in o.records)


def test_relaxed_strategy_is_lossy():
    """Lemma 4: RM prunes vertices that would have moved; the result differs from the baseline."""
    g = gg.make("lfr_small")
    base = oracle.louvain(g, prune=NONE)
    rm = oracle.louvain(g, prune=RM, check=True, trace=1)
    assert sum(r.n_fn for r in rm.records) > 0
    assert not np.array_equal(rm.labels, base.labels)
    assert abs(rm.Q - base.Q) < 0.02                  # a small loss (Table 3 scale)


def _neighbours(g, v):
    return g.col[g.row_ptr[v]:g.row_ptr[v + 1]]


@pytest.mark.parametrize("gi", [0, 1, 2, 3])
def test_iteration1_pruned_sets_from_definitions(gi):
    """Level 0, iteration 1: every strategy starts from the same state (iteration 0 evaluates
    every vertex for gamma = 1: c15), so the SM / RM pruned counts follow from the iteration-0
    moves by the definitions of P:157 / P:163, and MG+RM prunes MG's set united with RM's."""
    g = graphs()[gi]
    recs = {m: oracle.louvain(g, prune=m, trace=2, max_levels=1, max_iters=2).records for m in (NONE, MG, SM, RM, MGRM)}
    assert all(len(r) == 2 for r in recs.values())
    lab0 = recs[NONE][0].labels                       # labels after iteration 0
    for m in (MG, SM, RM, MGRM):
        assert np.array_equal(recs[m][0].labels, lab0) and recs[m][0].n_pruned == 0
    n = g.n
    start = np.arange(n)
    moved = lab0 != start
    changed = set(start[moved].tolist()) | set(lab0[moved].tolist())
    deg = np.diff(g.row_ptr)
    sm = rm = 0
    rm_set = set()
    for v in range(n):
        if deg[v] == 0:
            continue
        nb = _neighbours(g, v)
        if lab0[v] not in changed and not any(lab0[u] in changed for u in nb):
            sm += 1
        if not any(moved[u] for u in nb if u != v):
            rm += 1
            rm_set.add(v)
    assert recs[SM][1].n_pruned == sm
    assert recs[RM][1].n_pruned == rm
    mg_p, both_p = recs[MG][1].n_pruned, recs[MGRM][1].n_pruned
    assert max(mg_p, rm) <= both_p <= mg_p + rm


def test_invalid_strategy_rejected():
    o = oracle.louvain(gg.karate(), prune=5)
    assert o.status == 1
