"""Host-side logic of the N>1 path on CPU with a world_size-2 gloo group:
edge-balanced partition, the local-rows slicing each rank hands to
gala_graph_from_csr_dist, the 128-byte uid broadcast (bench.py does the same
with an NCCL group), and bench.py's max-over-ranks timing reduction."""
import os
import socket

import numpy as np
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen as gg
import paper_conf_ppopp_wangllwm00z25_b200 as gala


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import torch
    g = gg.make("lfr_small")
    bounds = gala.partition_ranges(g.row_ptr, world)
    lrp, lcol, lw = gala.local_rows(g.row_ptr, g.col, g.w, int(bounds[rank]), int(bounds[rank + 1]))
    # every rank's slice, gathered, must rebuild the global CSR exactly
    pieces = [None] * world
    dist.all_gather_object(pieces, (int(bounds[rank]), lrp.tolist(), lcol.tolist()))
    rp = [0]
    col = []
    for v0, r, c in sorted(pieces):
        base = rp[-1]
        rp.extend([x + base for x in r[1:]])
        col.extend(c)
    ok_csr = np.array_equal(np.array(rp), g.row_ptr) and np.array_equal(np.array(col, dtype=np.int32), g.col)
    # uid broadcast exactly as bench.py does it
    uid = [gala.loopback_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(uid, src=0)
    # max-over-ranks of the timed region (bench.py reduces elapsed ms with MAX)
    from bench import max_over_ranks
    t = max_over_ranks(10.0 + rank)
    loads = (g.row_ptr[bounds[1:]] - g.row_ptr[bounds[:-1]]).tolist()
    q.put((rank, ok_csr, len(uid[0]), uid[0][:8], t, loads))
    dist.destroy_process_group()


def test_gloo_world2_partition_uid_and_timing():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok_csr, ulen, head, t, loads in res:
        assert ok_csr
        assert ulen == 128 and head == b"GALALOOP"
        assert t == 11.0                       # max over ranks
        assert max(loads) - min(loads) <= 2 * 200 + 1   # edge-balanced within one max row


def _worker_shared(rank, world, port, q, tmp):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), GALA_SHARED_GRAPH_DIR=tmp)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from bench import shared_graph
    g, cleanup = shared_graph("lfr_small", rank, world)
    ref = gg.make("lfr_small")
    same = (np.array_equal(np.asarray(g.row_ptr), ref.row_ptr) and np.array_equal(np.asarray(g.col), ref.col)
            and np.array_equal(np.asarray(g.truth), ref.truth) and g.n == ref.n and g.nnz == ref.nnz)
    bounds = gala.partition_ranges(g.row_ptr, world)
    lrp, lcol, _ = gala.local_rows(g.row_ptr, g.col, g.w, int(bounds[rank]), int(bounds[rank + 1]))
    cleanup()
    left = os.listdir(tmp)
    q.put((rank, same, int(lrp[-1]) == len(lcol), left))
    dist.destroy_process_group()


def test_gloo_world2_shared_graph(tmp_path):
    """bench.py's N-rank graph loading: rank 0 generates, the other ranks map its arrays; every
    rank sees the generator's graph exactly and the scratch directory is gone afterwards."""
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker_shared, args=(r, world, port, q, str(tmp_path))) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, same, rows_ok, left in res:
        assert same and rows_ok
    assert os.listdir(str(tmp_path)) == []
