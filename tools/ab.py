"""A/B timing of option sets on one workload (median of N runs, graph mode)."""
import sys, json, statistics; sys.path.insert(0, '.')
import torch, graphgen as gg, paper_conf_ppopp_wangllwm00z25_b200 as gala
g = gg.make(sys.argv[1])
sets = json.loads(sys.argv[2])
stream = torch.cuda.Stream()
flush = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device="cuda")
for opts in sets:
    h = gala.Graph.from_graph(g, stream=stream.cuda_stream)
    for k, v in opts.items(): h.set_option(k, v)
    for _ in range(3): h.run()
    ts = []
    for _ in range(9):
        with torch.cuda.stream(stream): flush.add_(1)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream); h.run(); e1.record(stream); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    h.set_option("timing", 1); h.set_option("cuda_graph", 0)
    h.run()
    ks = {k: round(v["ms"], 3) for k, v in h.kernel_stats().items() if v["ms"] > 0.05}
    print(f"{json.dumps(opts):60s} median {statistics.median(ts):7.3f} ms  {ks}", flush=True)
    h.free()
