"""Per-level breakdown of one workload: graph-mode run time, then a stepwise
timed run (per-level phase-1/phase-2 ms, per-kernel-class ms)."""
import json, sys, time; sys.path.insert(0, '.')
import torch, graphgen as gg, paper_conf_ppopp_wangllwm00z25_b200 as gala
cfg = sys.argv[1]
opts = json.loads(sys.argv[2]) if len(sys.argv) > 2 else {}
t = time.time(); g = gg.make(cfg); print(f"{cfg}: n={g.n} nnz={g.nnz} gen {time.time()-t:.1f}s", flush=True)
stream = torch.cuda.Stream()
h = gala.Graph.from_graph(g, stream=stream.cuda_stream)
for k, v in opts.items(): h.set_option(k, v)
ts = []
for i in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream); h.run(); e1.record(stream); torch.cuda.synchronize()
    ts.append(round(e0.elapsed_time(e1), 2))
print("graph-mode run ms", ts, "Q", round(h.modularity(), 6), flush=True)
h.set_option("timing", 1); h.set_option("cuda_graph", 0)
h.run()
st = h.stats()
for i, l in enumerate(st["levels"]):
    print(f"L{i}: n={l['n']} nnz={l['nnz']} iters={l['iters']} maxdeg={l['maxdeg']} mode={l['mode']} "
          f"p1={l['ms_phase1']:.2f} p2={l['ms_phase2']:.2f} scanned={l['edges_scanned']}")
print({k: round(v["ms"], 3) for k, v in h.kernel_stats().items() if v["ms"] > 0.01})
