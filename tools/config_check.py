"""Run one BASELINE config on the GPU (timed) and optionally the oracle; compare."""
import sys, time, json; sys.path.insert(0, '.')
import numpy as np, torch
import graphgen as gg
import paper_conf_ppopp_wangllwm00z25_b200 as gala
name = sys.argv[1]
do_oracle = len(sys.argv) > 2 and sys.argv[2] == "oracle"
t = time.time(); g = gg.make(name); tg = time.time() - t
d = g.degrees()
print(f"{name}: n={g.n} nnz={g.nnz} maxdeg={d.max()} isolated={(d == 0).sum()} gen={tg:.1f}s", flush=True)
h = gala.Graph.from_graph(g)
h.set_option("trace", 1)
import os
if os.environ.get("GALA_VERBOSE"): h.set_option("verbose", 1)
for i in range(3):
    torch.cuda.synchronize(); t = time.time(); h.run(); torch.cuda.synchronize(); dt = time.time() - t
st = h.stats()
lab = h.communities(); Q = h.modularity(); N = h.numerator()[0]
print(f"gpu: {dt*1e3:.2f} ms run_ms={st['run_ms']:.2f} Q={Q:.6f} k={lab.max()+1}", flush=True)
print(" levels", [(l['n'], l['nnz'], l['iters'], l['maxdeg'], l['mode'], round(l['ms_phase1'], 2), round(l['ms_phase2'], 2)) for l in st['levels']], flush=True)
tr = h.trace()
if do_oracle:
    import oracle
    t = time.time(); o = oracle.louvain(g, prune=True, trace=1); to = time.time() - t
    same = np.array_equal(o.labels, lab) and o.N == N and len(o.records) == len(tr) and all(
        x.N == y["N"] and x.n_moved == y["n_moved"] for x, y in zip(o.records, tr))
    print(f"oracle: {to:.1f}s Q={o.Q:.6f} parity={'OK' if same else 'MISMATCH'}", flush=True)
