"""Pins of the CPU oracle against things other than itself.

Every test here is CPU-only.  The oracle (oracle/gala_oracle.c) is checked
against: literature values for the karate club, networkx's independent
modularity routine, closed forms (singletons, all-in-one, ring of cliques),
the brute-force optimum over all set partitions of small graphs, and
identities between two different formulas (Eq. 1 vs Eq. 2).
"""
import json
import os
import subprocess
import sys

import networkx as nx
import numpy as np
import pytest

import graphgen as gg
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def to_nx(g, weighted=True):
    G = nx.Graph()
    G.add_nodes_from(range(g.n))
    w = g.weights()
    for v in range(g.n):
        for e in range(g.row_ptr[v], g.row_ptr[v + 1]):
            u = int(g.col[e])
            if u > v:
                G.add_edge(v, u, weight=int(w[e]))
    return G


def nx_Q(g, labels, gamma=1.0):
    """networkx modularity (independent implementation of Eq. 1 with resolution)."""
    G = to_nx(g)
    comms = {}
    for v, c in enumerate(labels):
        comms.setdefault(int(c), set()).add(v)
    return nx.community.modularity(G, list(comms.values()), weight="weight", resolution=gamma)


# --------------------------------------------------------------------- P1
def test_karate_edge_list_matches_networkx_and_literature(golden_dir):
    gold = json.load(open(os.path.join(golden_dir, "karate.json")))
    g = gg.karate()
    assert g.n == gold["n"] and g.nnz == 2 * gold["m"]
    assert list(np.diff(g.row_ptr)) == gold["degree_sequence"]
    G = nx.karate_club_graph()
    ours = {(min(a, b), max(a, b)) for a, b in zip(np.repeat(np.arange(g.n), np.diff(g.row_ptr)), g.col)}
    theirs = {(min(a, b), max(a, b)) for a, b in G.edges()}
    assert ours == theirs


def test_karate_optimum_partition_literature_value(golden_dir):
    gold = json.load(open(os.path.join(golden_dir, "karate.json")))
    g = gg.karate()
    lab = np.zeros(34, dtype=np.int32)
    for i, part in enumerate(gold["optimum"]["partition"]):
        lab[part] = i
    Q = oracle.modularity(g, lab)
    assert round(Q, 4) == gold["optimum"]["Q_4dp"]
    W, N = oracle.partition_numerator(g, lab)
    assert W == 156 and N == 10216          # Q = 10216 / 156^2
    r = oracle.louvain(g)
    assert r.status == 0
    assert r.Q <= Q + 1e-15                  # Louvain cannot beat the proven optimum
    assert r.Q > 0.40


def test_karate_closed_forms():
    g = gg.karate()
    d = np.diff(g.row_ptr)
    W, N = oracle.partition_numerator(g, np.arange(34, dtype=np.int32))
    assert N == -int((d.astype(np.int64) ** 2).sum()) == -1212     # singletons: Q = -sum (d/2m)^2
    W, N = oracle.partition_numerator(g, np.zeros(34, dtype=np.int32))
    assert N == 0                                                    # all in one: Q = 1 - 1


# --------------------------------------------------------------------- modularity vs networkx
@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("gamma", [1.0, 0.5, 1.5, 2.0])
def test_modularity_matches_networkx(seed, gamma):
    rng = np.random.default_rng(seed)
    g = gg.random_graph(int(rng.integers(5, 40)), int(rng.integers(5, 120)), seed=seed, max_w=5)
    for _ in range(3):
        k = int(rng.integers(1, g.n + 1))
        lab = rng.integers(0, k, size=g.n).astype(np.int32)
        assert oracle.modularity(g, lab, gamma) == pytest.approx(nx_Q(g, lab, gamma), abs=1e-12)


@pytest.mark.parametrize("r,s", [(3, 3), (4, 3), (3, 4), (5, 4), (6, 5)])
def test_ring_of_cliques_closed_form(r, s):
    g = gg.ring_of_cliques(r, s)
    lab = np.repeat(np.arange(r), s).astype(np.int32)
    expected = 1 - 2 / (s * (s - 1) + 2) - 1 / r
    assert oracle.modularity(g, lab) == pytest.approx(expected, abs=1e-14)
    res = oracle.louvain(g)
    assert res.Q == pytest.approx(expected, abs=1e-14)
    assert res.k == r


def test_gamma_quantisation():
    assert oracle.gamma_pq(1.0) == (1, 1)
    assert oracle.gamma_pq(0.5) == (1, 2)
    assert oracle.gamma_pq(1.5) == (3, 2)
    assert oracle.gamma_pq(0.3) == (19661, 65536)


# --------------------------------------------------------------------- P2 gain identity
@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("gamma", [1.0, 0.5, 1.5, 5.0, 0.25])
def test_gain_closed_form_equals_bruteforce_difference(seed, gamma):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(4, 30))
    g = gg.random_graph(n, int(rng.integers(n, 4 * n)), seed=100 + seed, max_w=4,
                        self_loops=int(rng.integers(0, 4)))
    for _ in range(12):
        lab = rng.integers(0, int(rng.integers(1, n + 1)), size=n).astype(np.int32)
        v = int(rng.integers(0, n))
        target = int(rng.integers(0, n))
        _, N0 = oracle.partition_numerator(g, lab, gamma)
        lab2 = lab.copy()
        lab2[v] = target
        _, N1 = oracle.partition_numerator(g, lab2, gamma)
        assert N1 - N0 == oracle.move_gain2(g, lab, v, target, gamma)


# --------------------------------------------------------------------- P3 iteration-1 closed form
def iteration1_prediction(g, gamma=1.0):
    """Level 0, singletons, no self loops: v -> argmax_u (qW w(v,u) - p d(u) d(v)) (lowest id on
    ties) iff that score > 0 (stay = 0) and u* < v (both singletons: swap suppression)."""
    p, q = oracle.gamma_pq(gamma)
    d = np.zeros(g.n, dtype=object)
    w = g.weights()
    for v in range(g.n):
        d[v] = int(w[g.row_ptr[v]:g.row_ptr[v + 1]].sum())
    W = int(sum(d))
    lab = np.arange(g.n, dtype=np.int32)
    for v in range(g.n):
        best, bs = v, 0
        for e in range(g.row_ptr[v], g.row_ptr[v + 1]):
            u = int(g.col[e])
            sc = q * W * int(w[e]) - p * d[u] * d[v]
            if sc > bs or (sc == bs and best != v and u < best):
                best, bs = u, sc
        if best != v and best < v:
            lab[v] = best
    return lab


def test_iteration1_closed_form_karate():
    g = gg.karate()
    pred = iteration1_prediction(g)
    r = oracle.louvain(g, trace=2)
    first = r.records[0]
    assert first.level == 0 and first.iter == 0
    assert np.array_equal(first.labels, pred)
    assert int((pred != np.arange(34)).sum()) == 17 == first.n_moved
    # N after iteration 1 from networkx's modularity of the predicted partition
    assert first.N == round(nx_Q(g, pred) * 156 * 156) == 3330


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("gamma", [1.0, 0.5, 2.0])
def test_iteration1_closed_form_random(seed, gamma):
    g = gg.random_graph(60, 200, seed=200 + seed, max_w=3)
    r = oracle.louvain(g, gamma=gamma, trace=2)
    assert np.array_equal(r.records[0].labels, iteration1_prediction(g, gamma))


def test_tie_break_lowest_id():
    # 2 is adjacent to 0 and 1 (both degree 1): equal gains -> joins the lower id 0.
    g = gg.build_csr(3, np.array([2, 2]), np.array([0, 1]))
    r = oracle.louvain(g, trace=2, max_levels=1)
    assert list(r.records[0].labels) == [0, 1, 0]


# --------------------------------------------------------------------- P4 invariants + trace Q
@pytest.mark.parametrize("name", ["karate", "lfr_small"])
def test_levels_preserve_N_and_trace_matches_networkx(name):
    g = gg.make(name)
    r = oracle.louvain(g, trace=2)
    assert r.status == 0
    for a, b in zip(r.levels, r.levels[1:]):
        assert b.N_start == a.N_end                      # coarsening preserves Q exactly
        assert b.n < a.n
    assert r.N == r.levels[-1].N_end
    assert r.Q == pytest.approx(nx_Q(g, r.labels), abs=1e-12)
    # level-0 trace N values against networkx modularity of the snapshot labels
    W = r.W
    for rec in r.records:
        if rec.level == 0 and rec.iter < 4:
            assert rec.N / (W * W) == pytest.approx(nx_Q(g, rec.labels), abs=1e-12)
    # canonical labels: ids 0..k-1 in order of smallest member
    seen = []
    for c in r.labels:
        if c not in seen:
            seen.append(c)
    assert seen == list(range(r.k))


# --------------------------------------------------------------------- P5 pruning
@pytest.mark.parametrize("seed", range(20))
def test_pruning_on_equals_off_and_no_false_negatives(seed):
    rng = np.random.default_rng(300 + seed)
    n = int(rng.integers(5, 80))
    g = gg.random_graph(n, int(rng.integers(n, 5 * n)), seed=300 + seed, max_w=int(rng.integers(1, 4)),
                        self_loops=int(rng.integers(0, 5)))
    gamma = [1.0, 0.5, 1.5, 5.0, 0.25][seed % 5]
    a = oracle.louvain(g, gamma=gamma, trace=2)
    b = oracle.louvain(g, gamma=gamma, trace=2, prune=True, check=True)
    assert a.status == 0 and b.status == 0
    assert len(a.records) == len(b.records)
    for x, y in zip(a.records, b.records):
        assert np.array_equal(x.labels, y.labels) and x.N == y.N
        assert y.n_fn == 0                                 # Theorem 6: MG has no false negatives
    assert np.array_equal(a.labels, b.labels)


def test_pruning_lfr_small_prunes_and_matches():
    g = gg.make("lfr_small")
    a = oracle.louvain(g, trace=2)
    b = oracle.louvain(g, trace=2, prune=True, check=True)
    assert np.array_equal(a.labels, b.labels)
    assert sum(x.n_fn for x in b.records) == 0
    assert sum(x.n_pruned for x in b.records) > 0
    for x, y in zip(a.records, b.records):
        assert np.array_equal(x.labels, y.labels)


# --------------------------------------------------------------------- P6 brute force
def all_partitions(n):
    """Restricted growth strings of length n (all set partitions)."""
    out = [[0]]
    for i in range(1, n):
        nxt = []
        for p in out:
            m = max(p)
            for c in range(m + 2):
                nxt.append(p + [c])
        out = nxt
    return np.array(out, dtype=np.int64)


def brute_force_Qmax(g, gamma=1.0):
    P = all_partitions(g.n)
    w = g.weights().astype(np.float64)
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    W = w.sum()
    inside = (P[:, src] == P[:, g.col]).astype(np.float64) @ w
    d = np.zeros(g.n)
    np.add.at(d, src, w)
    onehot = (P[:, :, None] == np.arange(g.n)[None, None, :]).astype(np.float64)
    DV = np.einsum("pvc,v->pc", onehot, d)
    Q = inside / W - gamma * (DV ** 2).sum(1) / W ** 2
    i = int(np.argmax(Q))
    return Q[i], P[i]


@pytest.mark.parametrize("seed", range(8))
def test_louvain_below_bruteforce_optimum(seed):
    rng = np.random.default_rng(400 + seed)
    n = int(rng.integers(5, 10))
    g = gg.random_graph(n, int(rng.integers(n, 3 * n)), seed=400 + seed, max_w=3)
    qmax, pbest = brute_force_Qmax(g)
    assert qmax == pytest.approx(nx_Q(g, pbest), abs=1e-12)   # brute-force Q is networkx's Q
    r = oracle.louvain(g)
    assert r.Q <= qmax + 1e-12
    assert r.Q == pytest.approx(nx_Q(g, r.labels), abs=1e-12)


@pytest.mark.parametrize("r,s,N_opt,W", [(2, 4, 288, 24), (3, 3, 240, 24), (4, 3, 512, 32)])
def test_small_bruteforce_optima_reached(r, s, N_opt, W):
    if r == 2:   # two disjoint K4 (no ring edge)
        src, dst = [], []
        for base in (0, 4):
            for a in range(4):
                for b in range(a + 1, 4):
                    src.append(base + a)
                    dst.append(base + b)
        g = gg.build_csr(8, np.array(src), np.array(dst))
    else:
        g = gg.ring_of_cliques(r, s)
    if g.n <= 10:
        qmax, _ = brute_force_Qmax(g)
        assert qmax == pytest.approx(N_opt / W ** 2, abs=1e-12)
    res = oracle.louvain(g)
    assert res.W == W and res.N == N_opt


# --------------------------------------------------------------------- degenerate inputs
def test_degenerate_inputs():
    empty = gg.build_csr(5, np.array([], dtype=np.int64), np.array([], dtype=np.int64))
    r = oracle.louvain(empty)
    assert r.status == 0 and r.Q == 0.0 and list(r.labels) == list(range(5))
    single = gg.build_csr(2, np.array([0]), np.array([1]))
    r = oracle.louvain(single)
    assert list(r.labels) == [0, 0] and r.Q == pytest.approx(0.0)
    loops = gg.build_csr(3, np.array([0, 1, 1]), np.array([0, 1, 2]), np.array([3, 2, 1]), keep_self_loops=True)
    r = oracle.louvain(loops)
    assert r.status == 0
    assert r.Q == pytest.approx(nx_Q_selfloop(loops, r.labels), abs=1e-12)


def nx_Q_selfloop(g, labels):
    """networkx counts a self loop twice in the degree and once in the internal weight; our
    convention stores it once and counts it once in both.  Giving networkx half the loop weight
    makes the two definitions coincide (degree w, m = W/2, internal 2*(w/2) = w)."""
    G = nx.Graph()
    G.add_nodes_from(range(g.n))
    w = g.weights()
    for v in range(g.n):
        for e in range(g.row_ptr[v], g.row_ptr[v + 1]):
            u = int(g.col[e])
            if u > v:
                G.add_edge(v, u, weight=float(w[e]))
            elif u == v:
                G.add_edge(v, v, weight=float(w[e]) / 2)
    comms = {}
    for v, c in enumerate(labels):
        comms.setdefault(int(c), set()).add(v)
    return nx.community.modularity(G, list(comms.values()), weight="weight")


@pytest.mark.parametrize("seed", range(5))
def test_modularity_with_self_loops_matches_networkx(seed):
    rng = np.random.default_rng(500 + seed)
    g = gg.random_graph(20, 60, seed=500 + seed, max_w=4, self_loops=5)
    for _ in range(3):
        lab = rng.integers(0, 6, size=g.n).astype(np.int32)
        assert oracle.modularity(g, lab) == pytest.approx(nx_Q_selfloop(g, lab), abs=1e-12)


def test_invalid_tol_rejected():
    g = gg.karate()
    assert oracle.louvain(g, tol=0.0).status == 1


# --------------------------------------------------------------------- P7 thread independence
def test_thread_count_independence():
    code = ("import sys; sys.path.insert(0, %r); import graphgen as gg, oracle, hashlib;"
            "r = oracle.louvain(gg.make('lfr_small'), trace=2, prune=True);"
            "h = hashlib.sha256(b''.join(x.labels.tobytes() for x in r.records)).hexdigest();"
            "print(h, r.N)") % ROOT
    outs = []
    for t in ("1", "4"):
        env = dict(os.environ, OMP_NUM_THREADS=t)
        outs.append(subprocess.check_output([sys.executable, "-c", code], env=env, text=True).strip())
    assert outs[0] == outs[1]
