import sys, time; sys.path.insert(0,'.')
import numpy as np, torch, graphgen as gg, paper_conf_ppopp_wangllwm00z25_b200 as gala
g = gg.make(sys.argv[1] if len(sys.argv) > 1 else "lfr_small")
h1 = gala.Graph.from_graph(g).run()
rp = torch.from_numpy(g.row_ptr).cuda(); col = torch.from_numpy(g.col).cuda()
h2 = gala.Graph.from_csr(rp, col).run()
a, b = h1.communities(), h2.communities()
print("host vs device input equal:", np.array_equal(a, b), h1.stats()["W"], h2.stats()["W"], h1.stats()["nnz"], h2.stats()["nnz"])
s1, s2 = h1.stats(), h2.stats()
print([ (l['n'], l['iters'], l['maxdeg']) for l in s1['levels']], [(l['n'], l['iters'], l['maxdeg']) for l in s2['levels']])
for opts in [dict(cuda_graph=0), dict(cuda_graph=1), dict(cuda_graph=0, timing=1)]:
    h = gala.Graph.from_graph(g)
    for k, v in opts.items(): h.set_option(k, v)
    for i in range(4):
        torch.cuda.synchronize(); t = time.perf_counter(); h.run(); dt = time.perf_counter() - t
    st = h.stats()
    print(opts, f"wall {dt*1e3:.2f} ms run_ms {st['run_ms']:.2f}", [(round(l['ms_phase1'], 2), round(l['ms_phase2'], 2), l['iters']) for l in st['levels']])
