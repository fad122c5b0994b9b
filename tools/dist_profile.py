"""Dist path on one GPU, host-side and per-level timing: `world` ranks through the loopback comm
(threads), or world 1 through a real NCCL communicator (`nccl` as 3rd argument).
usage: tools/dist_profile.py <config> <world> [nccl] [verbose]"""
import sys, time, threading; sys.path.insert(0, '.')
import numpy as np, torch, graphgen as gg, paper_conf_ppopp_wangllwm00z25_b200 as gala
g = gg.make(sys.argv[1] if len(sys.argv) > 1 else "lfr1m")
world = int(sys.argv[2]) if len(sys.argv) > 2 else 1
nccl = len(sys.argv) > 3 and sys.argv[3] == "nccl"
verbose = "verbose" in sys.argv[3:]
bounds = gala.partition_ranges(g.row_ptr, world)
uid = gala.nccl_unique_id() if nccl else gala.loopback_unique_id()
res = [None] * world
def worker(r):
    lrp, lcol, lw = gala.local_rows(g.row_ptr, g.col, g.w, int(bounds[r]), int(bounds[r + 1]))
    h = gala.Graph.from_csr_dist(uid, r, world, 0, g.n, int(bounds[r]), int(bounds[r + 1]), lrp, lcol, lw)
    ts = []
    for i in range(4):
        if i == 3:
            h.set_option("timing", 1)
            if verbose: h.set_option("verbose", 1)
        t = time.time(); h.run(); ts.append(round(1e3 * (time.time() - t), 1))
    st = h.stats()
    res[r] = (ts, st["run_ms"], st["dist"], [(l["iters"], round(l["ms_phase1"], 2), round(l["ms_phase2"], 2)) for l in st["levels"]],
              {k: round(v["ms"], 3) for k, v in h.kernel_stats().items() if v["ms"] > 0.05})
ts = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
[t.start() for t in ts]; [t.join() for t in ts]
for r in res: print(r)
