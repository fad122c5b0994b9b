"""One gala_run on a workload, bracketed by cudaProfilerStart/Stop for
`ncu --profile-from-start off` (launch lists and full captures)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ppopp_wangllwm00z25_b200 as gala  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="lfr1m")
ap.add_argument("--warm", type=int, default=1)
ap.add_argument("--max-levels", type=int, default=0)
ap.add_argument("--cuda-graph", type=int, default=0, help="ncu cannot see kernels inside conditional graphs")
args = ap.parse_args()
g = gg.make(args.config)
h = gala.Graph.from_graph(g)
h.set_option("cuda_graph", args.cuda_graph)
for _ in range(args.warm):
    h.run(max_levels=args.max_levels)
torch.cuda.synchronize()
torch.cuda.profiler.start()
h.run(max_levels=args.max_levels)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
st = h.stats()
print({k: v for k, v in st.items() if k != "kernels"})
