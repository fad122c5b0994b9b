import sys, time, threading; sys.path.insert(0, '.')
import torch, graphgen as gg, paper_conf_ppopp_wangllwm00z25_b200 as gala
sys.path.insert(0, '.')
from bench import ClockSampler
g = gg.make(sys.argv[1] if len(sys.argv) > 1 else "lfr1m")
stream = torch.cuda.Stream()
h = gala.Graph.from_graph(g, stream=stream.cuda_stream)
flush = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device="cuda")
def steps(n, label):
    out = []
    for _ in range(n):
        with torch.cuda.stream(stream):
            flush.add_(1)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t = time.perf_counter()
        e0.record(stream); h.run(); e1.record(stream); torch.cuda.synchronize()
        out.append((round(e0.elapsed_time(e1), 2), round((time.perf_counter() - t) * 1e3, 2), round(h.stats()["run_ms"], 2)))
    print(label, out)
for opts in [dict(cuda_graph=1), dict(cuda_graph=0), dict(cuda_graph=1, singleton=0)]:
    for k, v in opts.items(): h.set_option(k, v)
    steps(3, f"warm {opts}")
    steps(6, f"plain {opts}")
    with ClockSampler(0):
        steps(6, f"sampler {opts}")
