"""Friendster-shaped graph (BASELINE.json configs[4]: 65.6M vertices, ~1.8B edges) on ONE B200:
generate it with the memory-lean host generator, run the full multi-level Louvain resident on the
device (graph mode, timed with CUDA events), and check the result against the CPU oracle on what
the oracle can compute at this size:
  * N of the final partition recomputed from the labels on the level-0 graph by the oracle
    (oracle.partition_numerator, Eq. 1 x q W^2) equals the library's exact numerator;
  * the first `--oracle-iters` iterations of level 0 (oracle run with max_levels=1,
    max_iters=k): labels, N, moved / active / pruned counts equal the library's trace.
Prints one JSON line (also the stats the bench line would carry)."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_wangllwm00z25_b200 as gala  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="friendster")
ap.add_argument("--runs", type=int, default=3)
ap.add_argument("--oracle-iters", type=int, default=2)
ap.add_argument("--opts", default="{}", help="JSON library options (set_option) for every run")
ap.add_argument("--verbose-last", action="store_true", help="option verbose=1 on the last timed run")
args = ap.parse_args()
out = {"config": args.config}
t = time.time()
g = gg.make(args.config)
out.update(gen_s=round(time.time() - t, 1), n=g.n, nnz=g.nnz, max_degree=int(g.degrees().max()), meta=g.meta)
print(json.dumps(out), flush=True)
stream = torch.cuda.Stream()
t = time.time()
h = gala.Graph.from_graph(g, stream=stream.cuda_stream)
torch.cuda.synchronize()
out["create_s"] = round(time.time() - t, 2)
for k, v in json.loads(args.opts).items():
    h.set_option(k, v)
ts = []
for i in range(args.runs):
    if args.verbose_last and i == args.runs - 1:
        h.set_option("verbose", 1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    h.run()
    e1.record(stream)
    torch.cuda.synchronize()
    ts.append(round(e0.elapsed_time(e1), 2))
st = h.stats()
lv0 = st["levels"][0]
out.update(run_ms=ts, levels=len(st["levels"]), iterations=sum(l["iters"] for l in st["levels"]),
           Q=h.modularity(), level0_ms_phase1=lv0["ms_phase1"], level0_active_edges=lv0["edges_scanned"],
           per_level=[{k: l[k] for k in ("n", "nnz", "iters", "ms_phase1", "ms_phase2")} for l in st["levels"]],
           device_used_gb=round((torch.cuda.mem_get_info()[1] - torch.cuda.mem_get_info()[0]) / 2**30, 1))
out["level0_gteps"] = lv0["edges_scanned"] / (lv0["ms_phase1"] * 1e-3) / 1e9
labels = h.communities()
N_gpu = h.numerator()[0]
t = time.time()
W, N_or = oracle.partition_numerator(g, labels)
out.update(N_match=(N_or == N_gpu), oracle_N_s=round(time.time() - t, 1))
print(json.dumps(out), flush=True)
if args.oracle_iters > 0:
    h.set_option("trace", 2)
    h.set_option("max_iters", args.oracle_iters)
    h.run(max_levels=1)
    tr = h.trace(labels=True)
    t = time.time()
    o = oracle.louvain(g, prune=True, max_levels=1, max_iters=args.oracle_iters, trace=2)
    out["oracle_iters_s"] = round(time.time() - t, 1)
    ok = len(tr) == len(o.records)
    for x, y in zip(o.records, tr):
        ok = ok and np.array_equal(x.labels, y["labels"]) and x.N == y["N"] and x.n_moved == y["n_moved"] \
            and x.n_active == y["n_active"] and x.n_pruned == y["n_pruned"]
    out["oracle_iters_match"] = bool(ok)
    out["oracle_iters"] = len(o.records)
print(json.dumps(out), flush=True)
