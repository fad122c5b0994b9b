"""Multi-GPU path (§8(e), a10) exercised on one GPU: `world` ranks run as threads of one
process through the loopback communicator (test hook); the partitioned algorithm (owned-range
prune/decide, dense/sparse label exchange, replicated Sigma_tot updates, summed counters,
distributed coarsening and re-partitioning) must reproduce the oracle bit for bit at every
iteration.  Each case runs in its own process (tests/dist_loopback_case.py).

Both backends: 0 = the fabric (device-resident iteration over peer memory, fabric.cuh:
per-sender dense/sparse slots, on-device barriers, mirror-block delta d', send-to-owner phase
2, CUDA-graph captured), 1 = host-driven collectives (one host round trip per iteration)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def check(graph, world, gamma=1.0, sync_mode=0, backend=0, trace=2, **opts):
    cfg = dict(graph=graph, world=world, gamma=gamma, sync_mode=sync_mode, backend=backend, trace=trace, opts=opts)
    env = dict(os.environ, CUDA_MODULE_LOADING="EAGER", GALA_FABRIC_TIMEOUT_MS="10000")
    r = subprocess.run([sys.executable, os.path.join(HERE, "dist_loopback_case.py"), json.dumps(cfg)],
                       capture_output=True, text=True, timeout=600, env=env)
    assert r.returncode == 0, (r.stdout[-2000:], r.stderr[-3000:])
    return json.loads(r.stdout.strip().splitlines()[-1])


@pytest.mark.parametrize("backend", [0, 1])
@pytest.mark.parametrize("world", [2, 3, 4])
def test_dist_lfr_small(world, backend):
    res = check("lfr_small", world, backend=backend)
    d = res["dist"][0]
    assert d["world"] == world and d["dense_iters"] + d["sparse_iters"] > 0


@pytest.mark.parametrize("backend", [0, 1])
@pytest.mark.parametrize("sync_mode", [1, 2])
def test_dist_forced_sync_modes(sync_mode, backend):
    d = check("rmat_small", 2, sync_mode=sync_mode, backend=backend)["dist"][0]
    if sync_mode == 1:   # forced dense: every exchange dense
        assert d["dense_iters"] > 0 and d["sparse_iters"] == 0
    elif backend == 1:   # forced sparse (host backend): every exchange sparse
        assert d["sparse_iters"] > 0 and d["dense_iters"] == 0
    else:                # fabric: sparse whenever the list fits the sender's slot
        assert d["sparse_iters"] > 0


@pytest.mark.parametrize("backend", [0, 1])
def test_dist_karate_and_weighted(backend):
    check("karate", 2, backend=backend)
    check(["random", 400, 3000, 77, 5, 4], 3, gamma=1.5, backend=backend)


@pytest.mark.parametrize("backend", [0, 1])
def test_dist_more_ranks_than_busy_rows(backend):
    check("karate", 4, backend=backend)


@pytest.mark.parametrize("backend", [0, 1])
def test_dist_hub_path(backend):
    """Rows split over blocks (hub path) on partitioned ranks, coarse levels included."""
    check("rmat_small", 3, backend=backend, bin_sub4=4, bin_sub8=8, bin_sub16=16, bin_sub32=32,
          bin_warp=32, bin_warp512=32, bin_block=32)


@pytest.mark.parametrize("delta", [0, 1, 2])
def test_dist_fabric_delta_modes(delta):
    """§3.5 across ranks: forced delta (mirror-block pushes every iteration), forced recompute
    and the adaptive choice give identical d' (the per-iteration N and labels match)."""
    check("lfr_small", 3, backend=0, delta_update=delta)


def test_dist_fabric_loopback_meets_on_host():
    """trace=1 would select the level's conditional CUDA graph; loopback ranks share one device,
    so the fabric barriers are host rendezvous and the level runs stepwise (no kernel ever
    spins on another rank's kernel).  Per-iteration N / counts still match the oracle; the
    graph-captured fabric iteration is covered through NCCL at world = 1 (test_dist_nccl.py)."""
    res = check("lfr_small", 4, backend=0, trace=1)
    assert any(u > 0 for u in res["us"])
