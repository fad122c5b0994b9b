import sys; sys.path.insert(0,'.')
import numpy as np, graphgen as gg, oracle, paper_conf_ppopp_wangllwm00z25_b200 as gala
g=gg.karate()
o=oracle.louvain(g, prune=True, trace=2)
print("oracle", [x.N for x in o.records])
for opts in [dict(cuda_graph=0), dict(cuda_graph=1), dict(cuda_graph=1, delta_update=0), dict(cuda_graph=1, delta_update=1),
             dict(cuda_graph=1, prune=0), dict(cuda_graph=1, max_iters=1), dict(cuda_graph=1, log_cap=2)]:
    h=gala.Graph.from_graph(g); h.set_option("trace", 1); h.set_option("check",1)
    for k,v in opts.items(): h.set_option(k,v)
    h.run(); tr=h.trace()
    print(opts, [y['N'] for y in tr], [y['delta_used'] for y in tr], h.stats()['dp_mismatch'])
