#!/usr/bin/env python
"""bench.py — GALA Louvain on B200: local-move GTEPS + end-to-end Louvain seconds + modularity.

Contract (driver): `python bench.py --gpus N --steps K --warmup W [--impl reference]` prints ONE
JSON line on rank 0.  A *step* is one full multi-level Louvain run (gala_run: every SURVEY.md §8(a)
row: init, MG prune/bin, DecideAndMove, apply, d' update, reductions, relabel, coarsen) over the
synthetic graph of the workload (default: the largest single-GPU config, BASELINE.json
configs[3], the Orkut-shaped graph 3.1M / 117.2M edges), restarting from singletons each step.
`--gpus N` without a launcher re-executes itself under torch.distributed.run (N ranks).

value  = local-move GTEPS: sum over the level-0 iterations of sum_{v active}
         deg(v) (the edges the decide kernels stream; pruned vertices are not counted) / level-0
         phase-1 device time (CUDA events inside the timed steps), whole job.  Inputs resident.
         Secondary: nominal GTEPS (iterations x nnz, all levels, credits pruning), full-run
         seconds (all levels + phase 2 = `ms_per_step`).
e2e    = the same metric with the level-0 phase-1 time replaced by the C-ABI call sequence from
         HOST buffers: gala_graph_from_csr (H2D) + gala_run + gala_get_communities (D2H).
roofline: dominant kernel class (by device time, CUDA events inside the library on its stream)
         algorithmic bytes / time vs MEASURED_PEAKS.json hbm_gbs; `phase1_roofline`: all level-0
         phase-1 algorithmic bytes / level-0 phase-1 time.
cpu_baseline: the CPU oracle (oracle/, plain C + OpenMP) on the same graph, all host cores;
         `oracle_1thread`: karate and LFR-1M full runs with one thread.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

WORKLOADS = {
    "lfr1m": "LFR planted partition 1M vertices / ~20M edges, mu=0.3 (BASELINE.json configs[1])",
    "karate": "Zachary karate club (BASELINE.json configs[0])",
    "rmat_lj": "R-MAT LiveJournal-shaped 4.8M / 69M (BASELINE.json configs[2])",
    "orkut": "Orkut-shaped LFR 3.1M / 117.2M edges, max degree 33.1k (BASELINE.json configs[3]; largest single-GPU config)",
    "friendster_q": "Friendster-shaped LFR at 1/4 scale, 16.4M / ~451M (BASELINE.json configs[4] shape on 1 GPU)",
    "friendster": "Friendster-shaped LFR 65.6M / 1.806B edges (BASELINE.json configs[4]) on ONE B200 (memory-lean "
                  "host generator, ~4 min on 16 cores; the 8-GPU partitioned run needs a multi-GPU box)",
    "lfr_small": "LFR 20k (test size)",
}
METRIC = "local-move GTEPS and end-to-end Louvain seconds at 1/2/4/8 B200; modularity Q"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)", d
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)", {}


class ClockSampler:
    """SM clock + throttle reasons sampled (NVML, 100 ms) during the timed region."""

    def __init__(self, device: int, period: float = 0.1):
        self.device, self.period = device, period
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()

    def __enter__(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            self.nv = nv
            self.h = nv.nvmlDeviceGetHandleByIndex(self.device)
            self.max_mhz = nv.nvmlDeviceGetMaxClockInfo(self.h, nv.NVML_CLOCK_SM)
            self._poll()
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        except Exception:
            self.nv = None
        return self

    def _poll(self):
        nv = self.nv
        self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
        r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        names = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
                 "sw_power_cap": 0x4}
        for k, bit in names.items():
            if r & bit:
                self.reasons.add(k)

    def _run(self):
        while not self._stop.wait(self.period):
            try:
                self._poll()
            except Exception:
                break

    def __exit__(self, *exc):
        self._stop.set()
        if self.nv:
            try:
                self._poll()
            except Exception:
                pass

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def max_over_ranks(x: float) -> float:
    """MAX of a host scalar over all ranks of the default process group (identity without one)."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return x
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def nominal_edges(stats: dict) -> int:
    return sum(lv["nominal_edges"] for lv in stats["levels"])


SAMPLE_NNZ = 300_000_000   # above this the oracle baseline is a bounded sample (first 2 iterations)


def oracle_baseline(g, steps=1):
    """The CPU oracle (test infrastructure) on the same graph, all host cores.  Graphs above
    SAMPLE_NNZ entries are timed on a bounded sample: level 0, first two iterations.  Level 0 is
    run (and timed) on its own first so its local-move GTEPS matches the GPU's `value`."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    times, l0_times = [], []
    res = None
    sample = g.nnz > SAMPLE_NNZ
    for _ in range(steps):
        t0 = time.perf_counter()
        r0 = oracle.louvain(g, prune=True, trace=3, max_levels=1, max_iters=2 if sample else 0)
        l0_times.append(time.perf_counter() - t0)
        if sample:
            res = r0
            times.append(l0_times[-1])
            continue
        t0 = time.perf_counter()
        res = oracle.louvain(g, prune=True, trace=1)
        times.append(time.perf_counter() - t0)
    deg = np.diff(g.row_ptr)
    # level-0 local-move edges: sum of deg(v) over the active vertices (d(v) > 0, not pruned)
    l0_active = sum(int(deg[(deg > 0) & ~rec.pruned].sum()) for rec in r0.records)
    edges = sum(lv.iters * lv.nnz for lv in res.levels)
    return dict(seconds=statistics.median(times), l0_seconds=statistics.median(l0_times), edges=edges,
                l0_active_edges=l0_active, cores=cores, Q=res.Q, N=res.N, labels=res.labels,
                iters=sum(lv.iters for lv in res.levels), sample=sample)


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle as the reference arm (rank 0 only), same metric: level-0
    local-move GTEPS (active edges / level-0 seconds); each step one oracle run of level 0
    (graphs above SAMPLE_NNZ: its first two iterations)."""
    if rank != 0:
        return
    import graphgen as gg
    import oracle
    g = gg.make(args.config)
    sample = g.nnz > SAMPLE_NNZ
    deg = np.diff(g.row_ptr)
    cores = len(os.sched_getaffinity(0))

    def one():
        t0 = time.perf_counter()
        r = oracle.louvain(g, prune=True, trace=3, max_levels=1, max_iters=2 if sample else 0)
        dt = time.perf_counter() - t0
        return dt, sum(int(deg[(deg > 0) & ~rec.pruned].sum()) for rec in r.records), r

    for _ in range(args.warmup):
        one()
    secs, edges, res = [], 0, None
    for _ in range(args.steps):
        dt, e, res = one()
        secs.append(dt)
        edges += e
    total = sum(secs)
    value = edges / total / 1e9
    what = "level 0, first 2 iterations" if sample else "level 0 to convergence"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": {"workload": args.config, "desc": WORKLOADS.get(args.config, ""), "n": g.n, "nnz": g.nnz,
                   "gamma": 1.0, "tol": 1e-6, "prune": 1, "parallelism": f"CPU oracle, {cores} threads",
                   "l2": "n/a (CPU)"},
        "value_def": "level-0 local-move GTEPS: sum over level-0 iterations of sum_{v active} deg(v) / level-0 seconds",
        "cpu_baseline": {"value": value, "unit": "GTEPS", "cores": cores, "kind": "oracle",
                         "sample": f"oracle {what} on {args.config} per step ({cpu_model()})"},
        "e2e": {"value": value, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def level0_edges_ms(stats: dict):
    """(active edges, phase-1 ms, algorithmic bytes) of level 0 of one run."""
    lv0 = stats["levels"][0]
    return lv0["edges_scanned"], lv0["ms_phase1"], lv0.get("alg_bytes", 0.0)


def oracle_1thread():
    """The oracle on karate and LFR-1M with ONE OpenMP thread (SURVEY.md §8(d) 'Timing'),
    in a subprocess (the thread count is fixed at OpenMP start-up)."""
    code = ("import json, time, graphgen as gg, oracle\n"
            "out = {}\n"
            "for name in ('karate', 'lfr1m'):\n"
            "    g = gg.make(name)\n"
            "    t = time.perf_counter(); r = oracle.louvain(g, prune=True, trace=1)\n"
            "    out[name] = {'seconds': time.perf_counter() - t, 'n': g.n, 'nnz': g.nnz, 'Q': r.Q}\n"
            "print(json.dumps(out))\n")
    env = dict(os.environ, OMP_NUM_THREADS="1", PYTHONPATH=ROOT)
    try:
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=600)
        return json.loads(r.stdout.strip().splitlines()[-1])
    except Exception as e:   # reporting only
        return {"error": str(e)[:200]}


def relaunch_distributed(args):
    """`--gpus N` (N > 1) started as a plain process: re-execute under torch.distributed.run so
    the N ranks exist (one process per GPU), forwarding rank 0's JSON line."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gala", choices=["gala", "reference"])
    ap.add_argument("--config", default="orkut", choices=sorted(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-oracle-1thread", action="store_true")
    ap.add_argument("--no-timing", action="store_true", help="skip the per-kernel-event (roofline) steps")
    ap.add_argument("--iter-jsonl", default=None, help="also write the per-iteration records to this JSONL file")
    ap.add_argument("--force-dist", action="store_true", help="use the multi-GPU (NCCL) path even at world size 1")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl != "reference" else args.warmup

    if args.gpus > 1 and "RANK" not in os.environ:
        sys.exit(relaunch_distributed(args))
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        return run_reference(args, rank, world)

    import torch
    import graphgen as gg
    import paper_conf_ppopp_wangllwm00z25_b200 as gala

    if world > 1 or args.force_dist:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        os.environ.setdefault("RANK", str(rank))
        os.environ.setdefault("WORLD_SIZE", str(world))
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        return run_dist(args, rank, world, local_rank)

    dev = 0
    torch.cuda.set_device(dev)
    stream = torch.cuda.Stream(device=dev)
    g = gg.make(args.config)
    peak, peak_src, peaks = load_peaks()

    # ------------------------------------------------------------ device-resident timing (value)
    h = gala.Graph.from_graph(g, device=dev, stream=stream.cuda_stream)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)   # > 126 MB L2

    def timed_steps(nsteps, timing):
        h.set_option("timing", int(timing))
        ms, edges, scanned, launches = [], 0, 0, 0
        l0 = [0, 0.0, 0.0]   # level-0 active edges, phase-1 ms, algorithmic bytes
        kst = {}
        for _ in range(nsteps):
            with torch.cuda.stream(stream):
                flush.add_(1)                                    # L2 flush between timed steps
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(stream)
            h.run()
            e1.record(stream)
            torch.cuda.synchronize()
            ms.append(e0.elapsed_time(e1))
            st = h.stats()
            edges += nominal_edges(st)
            scanned += sum(lv["edges_scanned"] for lv in st["levels"])
            for i, x in enumerate(level0_edges_ms(st)):
                l0[i] += x
            launches += st["kernel_launches"]
            if timing:
                for k, v in h.kernel_stats().items():
                    acc = kst.setdefault(k, dict(launches=0, ms=0.0, alg_bytes=0.0))
                    for f in acc:
                        acc[f] += v[f]
        return ms, edges, scanned, launches, kst, l0

    with ClockSampler(dev) as clk:
        timed_steps(args.warmup, False)          # warm-up: identical steps (flush included), untimed
        step_ms, edges, scanned, launches, _, l0 = timed_steps(args.steps, False)
    # per-kernel CUDA-event timing (stepwise launch mode) for the roofline, same workload
    inst_ms, _, _, _, kstats, _ = timed_steps(max(2, min(args.steps, 5)), not args.no_timing)
    labels = h.communities()
    Q = h.modularity()
    last_stats = h.stats()
    # per-iteration records (north star reporting) from one more (untimed) traced run:
    # pruned fraction = |inactive| / |{v : d(v) > 0}| = n_pruned / (n_active + n_pruned)
    h.set_option("trace", 1)
    h.set_option("timing", 0)
    h.run()
    pruned, iter_log = {}, []
    for r in h.trace():
        tot = r["n_active"] + r["n_pruned"]
        frac = round(r["n_pruned"] / tot, 4) if tot else 0.0
        pruned.setdefault(f"L{r['level']}", []).append(frac)
        iter_log.append({"level": r["level"], "iter": r["iter"], "n_level": r["n_level"], "active": r["n_active"],
                         "moved": r["n_moved"], "pruned": r["n_pruned"], "pruned_frac": frac,
                         "active_edges": r["edges_scanned"], "sync": "local", "alg_bytes": r["alg_bytes"],
                         "us": r["us"], "delta_dp": r["delta_used"]})
    h.set_option("trace", 0)
    h.free()
    if args.iter_jsonl:
        with open(args.iter_jsonl, "w") as f:
            for rec in iter_log:
                f.write(json.dumps(dict(rec, workload=args.config)) + "\n")
    total_s = sum(step_ms) / 1e3
    l0_edges, l0_ms, l0_bytes = l0
    value = l0_edges / (l0_ms / 1e3) / 1e9               # level-0 local-move GTEPS (active edges)

    # dominant kernel (by device time) roofline
    # dominant single-kernel class of the phase-1 hot path (phase2 / level_init are multi-kernel
    # regions with host syncs, reported in kernels_ms_per_step only)
    cand = {k: v for k, v in kstats.items() if k not in ("phase2", "level_init") and v["alg_bytes"] > 0}
    dom = max(cand.items(), key=lambda kv: kv[1]["ms"]) if cand else None
    roofline = None
    if dom and dom[1]["ms"] > 0:
        name, ks = dom
        achieved = ks["alg_bytes"] / (ks["ms"] / 1e3) / 1e9
        traffic = None
        tpath = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tpath):
            t = json.load(open(tpath))
            traffic = t.get(args.config, {}).get(name, {}).get("dram_bytes_per_launch")
        roofline = {"bound": "hbm", "kernel": name, "achieved": achieved, "peak": peak, "unit": "GB/s",
                    "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                    "alg_bytes_per_launch": ks["alg_bytes"] / max(ks["launches"], 1),
                    "avg_launch_us": 1e3 * ks["ms"] / max(ks["launches"], 1)}
    decide = {k: v for k, v in kstats.items() if k.startswith("decide")}
    dec_ms = sum(v["ms"] for v in decide.values())
    dec_by = sum(v["alg_bytes"] for v in decide.values())
    p1_achieved = l0_bytes / (l0_ms / 1e3) / 1e9 if l0_ms else None

    # ------------------------------------------------------------ e2e through the C ABI with host buffers
    # (the resident handle of the device-timed leg is released first: one graph on the device at a
    # time, as a user of the C ABI runs it; its parked pool serves the e2e handles)
    h.free()
    rp = torch.from_numpy(g.row_ptr).pin_memory()
    col = torch.from_numpy(g.col).pin_memory()
    lab_host = torch.empty(g.n, dtype=torch.int32).pin_memory()
    e2e_ms, e2e_edges, iters_total, e2e_parts = [], 0, 0, []
    import ctypes
    L = gala.lib()
    # create / run / free cycles need ~8 cycles before the adopted allocation cache stops growing
    # (profiles/r02/r02zk, r02zs: cycles 6-8 of a fresh sequence run 40-45 ms slower, in gala_run
    # only; every later cycle is steady): at least 8 untimed cycles, recorded in the line
    e2e_warm = max(args.warmup, 8)
    for i in range(e2e_warm + args.steps):
        with torch.cuda.stream(stream):
            flush.add_(1)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ec, er = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        hh = ctypes.c_void_p()
        gala._check(L.gala_graph_from_csr(g.n, rp.data_ptr(), col.data_ptr(), None, dev, stream.cuda_stream,
                                          ctypes.byref(hh)))
        ec.record(stream)
        gala._check(L.gala_run(hh, 1.0, 1e-6, 0))
        er.record(stream)
        k = ctypes.c_int64()
        gala._check(L.gala_get_communities(hh, lab_host.data_ptr(), g.n, ctypes.byref(k)))
        e1.record(stream)
        torch.cuda.synchronize()
        gh = gala.Graph(hh, g.n)
        st = gh.stats()
        gh.free()
        if i >= e2e_warm:
            e2e_ms.append(e0.elapsed_time(e1))
            e2e_parts.append((e0.elapsed_time(ec), ec.elapsed_time(er), er.elapsed_time(e1)))
            e2e_edges += level0_edges_ms(st)[0]
            iters_total = sum(lv["iters"] for lv in st["levels"])
    e2e_value = e2e_edges / (sum(e2e_ms) / 1e3) / 1e9
    h2d = g.row_ptr.nbytes + g.col.nbytes
    d2h = g.n * 4 + iters_total * 2 * 128

    # ------------------------------------------------------------ CPU oracle baseline
    cpu = None
    parity = None
    if not args.no_cpu_baseline:
        ob = oracle_baseline(g, 1)
        what = ("level 0, first 2 iterations of the oracle (prune on; bounded sample)" if ob["sample"]
                else "one full multi-level oracle run (prune on)")
        cpu = {"value": ob["l0_active_edges"] / ob["l0_seconds"] / 1e9, "unit": "GTEPS", "cores": ob["cores"],
               "kind": "oracle",
               "sample": f"{what} on {args.config}, level-0 local-move GTEPS over its {ob['l0_seconds']:.2f} s of "
                         f"level 0 ({ob['seconds']:.2f} s whole run; {cpu_model()})",
               "louvain_seconds": ob["seconds"]}
        # a bounded sample has no final labels to compare; the full-size parity test covers it
        parity = None if ob["sample"] else bool(np.array_equal(ob["labels"], labels))
    o1 = None if args.no_oracle_1thread else oracle_1thread()

    lv0 = last_stats["levels"][0]
    line = {
        "metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * total_s / args.steps, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "int64", "data": "synthetic",
        "config": {"workload": args.config, "desc": WORKLOADS.get(args.config, ""), "n": g.n, "nnz": g.nnz,
                   "max_degree": int(np.diff(g.row_ptr).max()) if g.n else 0,
                   "gamma": 1.0, "tol": 1e-6, "prune": 1, "parallelism": "1 GPU",
                   "l2": "flushed between timed steps (256 MB write)"},
        "value_def": "level-0 local-move GTEPS: sum over level-0 iterations of sum_{v active} deg(v) / level-0 "
                     "phase-1 device time",
        "louvain_seconds": total_s / args.steps,
        "level0_phase1_ms": l0_ms / args.steps,
        "level0_active_edges": l0_edges // args.steps,
        "nominal_gteps": edges / total_s / 1e9,
        "gteps_scanned_all_levels": scanned / total_s / 1e9,
        "step_ms": [round(x, 3) for x in step_ms],
        "modularity": Q,
        "nmi_vs_planted": (gala.nmi(torch.as_tensor(labels, dtype=torch.int32).cuda(),
                                    torch.as_tensor(g.truth, dtype=torch.int32).cuda())
                           if getattr(g, "truth", None) is not None else None),
        "pruned_fraction_per_iteration": pruned,
        "levels": len(last_stats["levels"]),
        "iterations": sum(lv["iters"] for lv in last_stats["levels"]),
        "per_level": [{"n": lv["n"], "nnz": lv["nnz"], "iters": lv["iters"], "ms_phase1": round(lv["ms_phase1"], 4),
                       "ms_phase2": round(lv["ms_phase2"], 4), "active_edges": lv["edges_scanned"]}
                      for lv in last_stats["levels"]],
        "iteration_log": iter_log,
        "phase1_roofline": {"bound": "hbm", "scope": "level 0, all phase-1 kernels", "achieved": p1_achieved,
                            "peak": peak, "unit": "GB/s", "frac": p1_achieved / peak if p1_achieved else None,
                            "alg_bytes": l0_bytes / args.steps},
        "phase2_roofline": ({"bound": "hbm", "achieved": kstats["phase2"]["alg_bytes"] / (kstats["phase2"]["ms"] / 1e3) / 1e9,
                             "peak": peak, "unit": "GB/s",
                             "frac": kstats["phase2"]["alg_bytes"] / (kstats["phase2"]["ms"] / 1e3) / 1e9 / peak,
                             "alg_bytes_per_run": kstats["phase2"]["alg_bytes"] / len(inst_ms)}
                            if kstats.get("phase2", {}).get("ms") else None),
        "phase2_share": sum(lv["ms_phase2"] for lv in last_stats["levels"]) / (total_s * 1e3 / args.steps),
        "decide_roofline": {"achieved": dec_by / (dec_ms / 1e3) / 1e9 if dec_ms else None, "peak": peak,
                            "frac": (dec_by / (dec_ms / 1e3) / 1e9) / peak if dec_ms else None,
                            "ms_per_step": dec_ms / max(len(inst_ms), 1)},
        "kernels_ms_per_step": {k: round(v["ms"] / len(inst_ms), 4) for k, v in sorted(kstats.items())},
        "instrumented_ms_per_step": sum(inst_ms) / len(inst_ms),
        "roofline": roofline,
        "cpu_baseline": cpu,
        "oracle_1thread": o1,
        "oracle_parity": parity,
        "e2e": {"value": e2e_value, "unit": "GTEPS", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "louvain_seconds": sum(e2e_ms) / 1e3 / len(e2e_ms), "step_ms": [round(x, 3) for x in e2e_ms],
                "warmup_cycles": e2e_warm,
                "median_create_run_labels_ms": [round(statistics.median(p[j] for p in e2e_parts), 3) for j in range(3)],
                "create_run_labels_ms_per_step": [[round(x, 2) for x in p] for p in e2e_parts]},
        "gpu_launches": launches,
        "clocks": clk.summary(),
    }
    print(json.dumps(line), flush=True)


def shared_graph(config: str, rank: int, world: int):
    """The workload graph on every rank of an N-process run, generated ONCE: rank 0 builds it and
    writes its arrays to a scratch directory, the other ranks map them read-only after a barrier
    (8 ranks generating the full Friendster shape side by side would need 8 x 30 GB of host
    memory and 8x the generator time).  Returns (CSR, cleanup) -- call cleanup() once every rank
    has copied its rows."""
    import shutil
    import tempfile
    import torch.distributed as dist
    import graphgen as gg
    base = os.environ.get("GALA_SHARED_GRAPH_DIR", tempfile.gettempdir())
    tag = [f"gala_graph_{config}_{os.getpid()}_{int(time.time() * 1e3)}" if rank == 0 else None]
    dist.broadcast_object_list(tag, src=0)
    d = os.path.join(base, tag[0])
    if rank == 0:
        g = gg.make(config)
        os.makedirs(d, exist_ok=True)
        np.save(os.path.join(d, "row_ptr.npy"), g.row_ptr)
        np.save(os.path.join(d, "col.npy"), np.asarray(g.col))
        if g.w is not None:
            np.save(os.path.join(d, "w.npy"), g.w)
        if g.truth is not None:
            np.save(os.path.join(d, "truth.npy"), g.truth)
    dist.barrier()
    if rank != 0:
        ld = lambda f: np.load(os.path.join(d, f), mmap_mode="r") if os.path.exists(os.path.join(d, f)) else None
        rp = ld("row_ptr.npy")
        g = gg.CSR(n=len(rp) - 1, row_ptr=rp, col=ld("col.npy"), w=ld("w.npy"), name=config, truth=ld("truth.npy"))

    def cleanup():
        dist.barrier()
        if rank == 0:
            shutil.rmtree(d, ignore_errors=True)
    return g, cleanup


def run_dist(args, rank, world, local_rank):
    """N > 1 (torchrun, one process per GPU): 1D edge-balanced vertex partition of the same graph,
    NCCL inside libgala for the per-iteration label / counter exchange (bootstrapped here with the
    torch process group).  Total work is fixed as N grows -> strong scaling."""
    import torch
    import torch.distributed as dist
    import graphgen as gg
    import paper_conf_ppopp_wangllwm00z25_b200 as gala

    dev = local_rank
    g, cleanup = shared_graph(args.config, rank, world)   # generated once (rank 0), mapped by the others
    bounds = gala.partition_ranges(g.row_ptr, world)
    v0, v1 = int(bounds[rank]), int(bounds[rank + 1])
    lrp, lcol, lw = gala.local_rows(g.row_ptr, g.col, g.w, v0, v1)
    cleanup()
    uid = [gala.nccl_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(uid, src=0)
    stream = torch.cuda.Stream(device=dev)
    h = gala.Graph.from_csr_dist(uid[0], rank, world, dev, g.n, v0, v1, lrp, lcol, lw, stream=stream.cuda_stream)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)
    peak, peak_src, _ = load_peaks()

    def step(fn):
        with torch.cuda.stream(stream):
            flush.add_(1)
        dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        torch.cuda.synchronize()
        dist.barrier()
        return max_over_ranks(e0.elapsed_time(e1))

    l0 = [0, 0.0]   # level-0 active edges (global), level-0 phase-1 ms (max over ranks)
    with ClockSampler(dev) as clk:
        for _ in range(args.warmup):
            step(h.run)
        step_ms = []
        for _ in range(args.steps):
            step_ms.append(step(h.run))
            e, ms, _ = level0_edges_ms(h.stats())
            l0[0] += e
            l0[1] += max_over_ranks(ms)
    st = h.stats()
    edges = nominal_edges(st)
    Q = h.modularity()
    labels = h.communities()
    total_s = sum(step_ms) / 1e3
    value = l0[0] / (l0[1] / 1e3) / 1e9              # level-0 local-move GTEPS, whole job

    # e2e through the C ABI from host buffers on every rank
    import ctypes
    e2e_ms = []
    L = gala.lib()
    lab_host = np.empty(g.n, dtype=np.int32)
    for i in range(args.warmup + args.steps):
        def e2e():   # same uid: the library reuses its cached NCCL communicator
            hh = gala.Graph.from_csr_dist(uid[0], rank, world, dev, g.n, v0, v1, lrp, lcol, lw,
                                          stream=stream.cuda_stream)
            hh.run()
            gala._check(L.gala_get_communities(hh._h, lab_host.ctypes.data_as(ctypes.c_void_p), g.n, None))
            hh.free()
        ms = step(e2e)
        if i >= args.warmup:
            e2e_ms.append(ms)
    e2e_value = (l0[0] / args.steps) * len(e2e_ms) / (sum(e2e_ms) / 1e3) / 1e9
    d = st.get("dist", {})
    line = {
        "metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * total_s / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": {"workload": args.config, "desc": WORKLOADS.get(args.config, ""), "n": g.n, "nnz": g.nnz,
                   "gamma": 1.0, "tol": 1e-6, "prune": 1, "parallelism": f"1D vertex partition x{world} (NCCL)",
                   "l2": "flushed between timed steps (256 MB write)"},
        "value_def": "level-0 local-move GTEPS: sum over level-0 iterations of sum_{v active} deg(v) / level-0 "
                     "phase-1 device time (max over ranks)",
        "louvain_seconds": total_s / args.steps,
        "level0_phase1_ms": l0[1] / args.steps,
        "nominal_gteps": edges * args.steps / total_s / 1e9,
        "step_ms": [round(x, 3) for x in step_ms],
        "modularity": Q,
        "levels": len(st["levels"]),
        "iterations": sum(lv["iters"] for lv in st["levels"]),
        "sync": {"dense_iters": d.get("dense_iters"), "sparse_iters": d.get("sparse_iters"),
                 "bytes_exchanged_per_run": d.get("bytes_exchanged")},
        "per_level": [{"n": lv["n"], "nnz": lv["nnz"], "iters": lv["iters"], "ms_phase1": round(lv["ms_phase1"], 4),
                       "ms_phase2": round(lv["ms_phase2"], 4)} for lv in st["levels"]],
        "roofline": None, "cpu_baseline": None,
        "e2e": {"value": e2e_value, "unit": "GTEPS", "h2d_bytes_per_step": int(lrp.nbytes + lcol.nbytes),
                "d2h_bytes_per_step": int(g.n * 4)},
        "gpu_launches": st["kernel_launches"],
        "clocks": clk.summary(),
    }
    h.free()
    if rank == 0:
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
