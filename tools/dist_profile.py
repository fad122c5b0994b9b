"""Dist path with the loopback comm on one GPU: host-side phase timing."""
import sys, time, threading; sys.path.insert(0, '.')
import numpy as np, torch, graphgen as gg, paper_conf_ppopp_wangllwm00z25_b200 as gala
g = gg.make(sys.argv[1] if len(sys.argv) > 1 else "lfr1m")
world = int(sys.argv[2]) if len(sys.argv) > 2 else 1
bounds = gala.partition_ranges(g.row_ptr, world)
uid = gala.loopback_unique_id()
res = [None] * world
def worker(r):
    lrp, lcol, lw = gala.local_rows(g.row_ptr, g.col, g.w, int(bounds[r]), int(bounds[r + 1]))
    h = gala.Graph.from_csr_dist(uid, r, world, 0, g.n, int(bounds[r]), int(bounds[r + 1]), lrp, lcol, lw)
    for i in range(3):
        if i == 2 and len(sys.argv) > 3: h.set_option("verbose", 1)
        t = time.time(); h.run(); dt = time.time() - t
    st = h.stats()
    res[r] = (dt, st["run_ms"], st["dist"], [(l["iters"], round(l["ms_phase1"], 2), round(l["ms_phase2"], 2)) for l in st["levels"]])
ts = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
[t.start() for t in ts]; [t.join() for t in ts]
for r in res: print(r)
