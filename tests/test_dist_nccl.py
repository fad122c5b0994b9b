"""The multi-GPU entry point through a REAL NCCL communicator (not the loopback test double):
world = 1 on the one GPU a test box has (NCCL refuses two ranks on one device).  The uid comes
from gala_nccl_unique_id, the communicator from ncclCommInitRank inside libgala, and the fabric
region goes through the NCCL path of share_region.  Both backends must reproduce the oracle at
every iteration and level (labels, N, moved / active / pruned counts)."""
import numpy as np
import pytest

import graphgen as gg
import oracle
import paper_conf_ppopp_wangllwm00z25_b200 as gala

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _graphs():
    return {"karate": gg.karate(), "lfr_small": gg.make("lfr_small"), "rmat_small": gg.make("rmat_small"),
            "weighted": gg.random_graph(400, 3000, seed=91, max_w=5, self_loops=4)}


GRAPHS = _graphs()


@pytest.mark.parametrize("backend", [0, 1])
@pytest.mark.parametrize("name", sorted(GRAPHS))
def test_nccl_world1_parity(name, backend):
    g = GRAPHS[name]
    o = oracle.louvain(g, prune=True, trace=2)
    uid = gala.nccl_unique_id()
    h = gala.Graph.from_csr_dist(uid, 0, 1, 0, g.n, 0, g.n, g.row_ptr, g.col, g.w)
    h.set_option("dist_backend", backend)
    h.set_option("trace", 2)
    h.run()
    tr = h.trace(labels=True)
    assert len(tr) == len(o.records)
    for x, y in zip(o.records, tr):
        assert (x.level, x.iter) == (y["level"], y["iter"])
        assert np.array_equal(x.labels, y["labels"])
        assert x.N == y["N"] and x.n_moved == y["n_moved"]
        assert x.n_active == y["n_active"] and x.n_pruned == y["n_pruned"]
    assert np.array_equal(h.communities(), o.labels)
    assert abs(h.modularity() - o.Q) <= 1e-9
    assert h.stats()["dist"]["world"] == 1
    h.free()


def test_nccl_world1_graph_mode_repeat_runs():
    """Graph-captured fabric iterations, the cached communicator reused by a second handle."""
    g = GRAPHS["lfr_small"]
    o = oracle.louvain(g, prune=True)
    uid = gala.nccl_unique_id()
    for _ in range(2):
        h = gala.Graph.from_csr_dist(uid, 0, 1, 0, g.n, 0, g.n, g.row_ptr, g.col, g.w)
        for _ in range(2):
            h.run()
            assert np.array_equal(h.communities(), o.labels)
        h.free()
