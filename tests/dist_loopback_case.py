"""One loopback multi-rank case (run by tests/test_dist_loopback.py in its own process).

argv[1]: JSON {"graph": name | ["random", n, m, seed, max_w, self_loops], "world": P,
               "gamma": g, "sync_mode": s, "backend": b, "trace": t, "opts": {...}}
Runs `world` ranks as threads of this process through the loopback communicator, compares
every rank with the oracle at every iteration (labels when trace >= 2, N, moved / active /
pruned counts) and prints one JSON line with the per-rank dist statistics.  Exit status 0 iff
everything matched.  Own process: a rank that fails cannot take the test session's CUDA
context down with it.
"""
import json
import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_MODULE_LOADING", "EAGER")
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_wangllwm00z25_b200 as gala  # noqa: E402


def make_graph(spec):
    if isinstance(spec, str):
        return gg.karate() if spec == "karate" else gg.make(spec)
    _, n, m, seed, max_w, loops = spec
    return gg.random_graph(n, m, seed=seed, max_w=max_w, self_loops=loops)


def main():
    cfg = json.loads(sys.argv[1])
    g = make_graph(cfg["graph"])
    world, gamma, trace = cfg["world"], cfg.get("gamma", 1.0), cfg.get("trace", 2)
    o = oracle.louvain(g, gamma=gamma, prune=True, trace=2)
    bounds = gala.partition_ranges(g.row_ptr, world)
    uid = gala.loopback_unique_id()
    out, err = [None] * world, []

    def worker(r):
        try:
            lrp, lcol, lw = gala.local_rows(g.row_ptr, g.col, g.w, bounds[r], bounds[r + 1])
            h = gala.Graph.from_csr_dist(uid, r, world, 0, g.n, int(bounds[r]), int(bounds[r + 1]), lrp, lcol, lw)
            h.set_option("trace", trace)
            h.set_option("sync_mode", cfg.get("sync_mode", 0))
            h.set_option("dist_backend", cfg.get("backend", 0))
            for k, v in cfg.get("opts", {}).items():
                h.set_option(k, v)
            h.run(gamma=gamma)
            out[r] = dict(labels=h.communities(), N=h.numerator()[0], trace=h.trace(labels=trace >= 2),
                          stats=h.stats())
            h.free()
        except Exception as e:  # noqa: BLE001
            err.append(f"rank {r}: {e}")

    ts = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=300)
    if err:
        print(json.dumps({"error": err}))
        sys.exit(1)
    for r in out:
        assert np.array_equal(r["labels"], o.labels), "final labels"
        assert r["N"] == o.N, "final N"
        assert len(r["trace"]) == len(o.records), "iteration count"
        for x, y in zip(o.records, r["trace"]):
            where = f"level {x.level} iter {x.iter}"
            assert (x.level, x.iter) == (y["level"], y["iter"]), where
            if trace >= 2:
                assert np.array_equal(x.labels, y["labels"]), where
            assert x.N == y["N"] and x.n_moved == y["n_moved"], where
            assert x.n_active == y["n_active"] and x.n_pruned == y["n_pruned"], where
    print(json.dumps({"dist": [r["stats"]["dist"] for r in out],
                      "us": [t["us"] for t in out[0]["trace"]]}))


if __name__ == "__main__":
    main()
