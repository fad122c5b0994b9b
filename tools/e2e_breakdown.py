"""Host-timed phases of one end-to-end C-ABI call sequence (bench.py's e2e leg): graph creation
from pinned host CSR, run, label copy-out, free.  usage: tools/e2e_breakdown.py <config>"""
import ctypes, sys, time; sys.path.insert(0, '.')
import torch, graphgen as gg, paper_conf_ppopp_wangllwm00z25_b200 as gala
g = gg.make(sys.argv[1] if len(sys.argv) > 1 else "lfr1m")
stream = torch.cuda.Stream()
rp = torch.from_numpy(g.row_ptr).pin_memory()
col = torch.from_numpy(g.col).pin_memory()
lab = torch.empty(g.n, dtype=torch.int32).pin_memory()
L = gala.lib()
NC = int(sys.argv[2]) if len(sys.argv) > 2 else 6
VERB = len(sys.argv) > 3
for i in range(NC):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    hh = ctypes.c_void_p()
    gala._check(L.gala_graph_from_csr(g.n, rp.data_ptr(), col.data_ptr(), None, 0, stream.cuda_stream, ctypes.byref(hh)))
    torch.cuda.synchronize(); t1 = time.perf_counter()
    if VERB:
        gala._check(L.gala_set_option(hh, b"verbose", 1))
    gala._check(L.gala_run(hh, 1.0, 1e-6, 0))
    torch.cuda.synchronize(); t2 = time.perf_counter()
    k = ctypes.c_int64()
    gala._check(L.gala_get_communities(hh, lab.data_ptr(), g.n, ctypes.byref(k)))
    torch.cuda.synchronize(); t3 = time.perf_counter()
    view = gala.Graph(hh, g.n)
    dev_ms = view.stats().get("run_ms", float("nan"))   # device time of the run
    view._h = None                                      # a view: freed below through the C ABI
    L.gala_graph_free(hh)
    torch.cuda.synchronize(); t4 = time.perf_counter()
    print(f"create {1e3*(t1-t0):7.2f} ms  run {1e3*(t2-t1):7.2f}  (device {dev_ms:7.2f})  labels {1e3*(t3-t2):6.2f}  free {1e3*(t4-t3):6.2f}", flush=True)
