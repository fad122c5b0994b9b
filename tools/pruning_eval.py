"""B200 evaluation of the pruning strategies and the paper's ablations (SURVEY.md §8(f)
NEXT #2-#4), one JSON object per line.

  strategies : for every strategy (none / MG / SM / RM / MG+RM): device time of a full
               multi-level run (graph mode, L2 flushed, median of 5), Q, iterations, the
               per-iteration inactive rate of level 0 (Fig. 7), and from an
               instrumented run (option prune_check) FNR / FPR over the level-0 iterations
               (Table 1); on LFR graphs NMI against the planted partition
               (Table 4).
  ablations  : Fig. 6 (no pruning + global-memory tables vs MG vs MG + memory
               management), Fig. 8 (B / P1 / P2 breakdown of DecideAndMove vs weight
               update), Fig. 9 (shuffle vs shared vs global tables for small rows;
               hierarchical vs unified vs global-only tables for long rows, with the shared-
               memory access / maintenance rates of Fig. 4).
usage: python tools/pruning_eval.py strategies|ablations CONFIG [CONFIG ...]
"""
import json
import statistics
import sys
import os

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ppopp_wangllwm00z25_b200 as gala  # noqa: E402

NAMES = {0: "none", 1: "MG", 2: "SM", 3: "RM", 4: "MG+RM"}
SMALL = ["bin_sub4", "bin_sub8", "bin_sub16", "bin_sub32"]
_flush = None


def timed(g, opts, reps=5):
    global _flush
    if _flush is None:
        _flush = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device="cuda")
    stream = torch.cuda.Stream()
    h = gala.Graph.from_graph(g, stream=stream.cuda_stream)
    for k, v in opts.items():
        h.set_option(k, v)
    h.run()
    ts = []
    for _ in range(reps):
        with torch.cuda.stream(stream):
            _flush.add_(1)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h.run()
        e1.record(stream)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return h, statistics.median(ts)


def kernel_ms(g, opts):
    h = gala.Graph.from_graph(g)
    for k, v in opts.items():
        h.set_option(k, v)
    h.set_option("timing", 1)
    h.set_option("cuda_graph", 0)
    h.run()
    ks = {k: round(v["ms"], 3) for k, v in h.kernel_stats().items() if v["ms"] > 0}
    st = h.stats()
    h.free()
    return ks, st


def nmi(truth, labels):
    from sklearn.metrics import normalized_mutual_info_score as f
    return dict(arithmetic=round(float(f(truth, labels, average_method="arithmetic")), 5),
                geometric=round(float(f(truth, labels, average_method="geometric")), 5))


def strategies(name):
    g = gg.make(name)
    for mode in range(5):
        h, ms = timed(g, dict(prune=mode))
        lab = h.communities()
        out = dict(kind="strategy", config=name, n=g.n, nnz=g.nnz, strategy=NAMES[mode], run_ms=round(ms, 3),
                   Q=round(h.modularity(), 6), levels=len(h.stats()["levels"]),
                   iterations=[lv["iters"] for lv in h.stats()["levels"]])
        h.free()
        h = gala.Graph.from_graph(g)
        h.set_option("prune", mode)
        h.set_option("prune_check", 1)
        h.set_option("trace", 1)
        h.run()
        tr = [r for r in h.trace() if r["level"] == 0]
        assert np.array_equal(h.communities(), lab), "instrumentation changed the result"
        h.free()
        fn = sum(r["n_fn"] for r in tr)
        fp = sum(r["n_fp"] for r in tr)
        tp = sum(r["n_moved"] for r in tr)
        tn = sum(r["n_pruned"] for r in tr) - fn
        out.update(level0_iterations=len(tr),
                   inactive_rate=[round(r["n_pruned"] / max(r["n_pruned"] + r["n_active"], 1), 4) for r in tr],
                   FNR=round(fn / max(fn + tp, 1), 5), FPR=round(fp / max(fp + tn, 1), 5),
                   false_negatives=fn, false_positives=fp)
        if getattr(g, "truth", None) is not None:
            out["NMI"] = nmi(g.truth, lab)
        print(json.dumps(out), flush=True)


def ablations(name):
    g = gg.make(name)
    # "global-memory tables": every row through the block kernel with the global-only table
    # (table_mode 1: every community in the block's global H1 -- the paper's baseline)
    glob = dict(bin_sub4=0, bin_sub8=0, bin_sub16=0, bin_sub32=0, bin_warp=0, bin_warp512=0, table_mode=1,
                block_split=0)
    rows = [
        ("fig6", "baseline: no pruning, global-memory tables", dict(glob, prune=0, delta_update=0)),
        ("fig6", "MG pruning, global-memory tables", dict(glob, prune=1)),
        ("fig6", "MG + memory management (default)", dict(prune=1)),
        ("fig8", "B: no pruning, d' recomputed", dict(prune=0, delta_update=0)),
        ("fig8", "P1: MG pruning, d' recomputed", dict(prune=1, delta_update=0)),
        ("fig8", "P2: MG pruning, d' delta-updated (default)", dict(prune=1)),
        ("fig9a", "rows <= 32: sub-warp shuffle (default)", dict()),
        ("fig9a", "rows <= 32: warp shared-memory hash", dict((k, 0) for k in SMALL)),
        ("fig9a", "all rows: block kernel, 64-slot H0 (global-memory hash)", glob),
        ("fig9b", "rows > 512: hierarchical smem H0 + global H1 (P:308; one block class)", dict(block_split=0)),
        ("fig9b", "rows > 512: unified smem + global, one hash (P:306)", dict(block_split=0, table_mode=2)),
        ("fig9b", "rows > 512: global-only (P:302)", dict(block_split=0, table_mode=1)),
        ("fig9b", "rows > 512: hierarchical, 1024-slot H0 (more spilling)", dict(block_split=0, hub_smem_slots=1024)),
        ("fig9b", "rows > 512: unified, 1024-slot H0", dict(block_split=0, hub_smem_slots=1024, table_mode=2)),
        ("fig9b", "rows > 512: multi-block hub path (global tables)", dict(bin_block=512)),
    ]
    for fig, label, opts in rows:
        h, ms = timed(g, opts, reps=3)
        Q = h.modularity()
        tb = h.stats()["table"]
        h.free()
        acc = tb["h0_access"] + tb["h1_access"]
        keys = tb["h0_keys"] + tb["h1_keys"]
        ks, st = kernel_ms(g, opts)
        dec = sum(v for k, v in ks.items() if k.startswith("decide"))
        print(json.dumps(dict(kind="ablation", figure=fig, config=name, variant=label, options=opts,
                              run_ms=round(ms, 3), Q=round(Q, 6), decide_ms=round(dec, 3),
                              smem_access_rate=round(tb["h0_access"] / acc, 4) if acc else None,
                              smem_maintenance_rate=round(tb["h0_keys"] / keys, 4) if keys else None,
                              dp_update_ms=ks.get("dp_update", 0.0), kernels_ms=ks)), flush=True)


if __name__ == "__main__":
    what = sys.argv[1]
    for c in sys.argv[2:]:
        (strategies if what == "strategies" else ablations)(c)
