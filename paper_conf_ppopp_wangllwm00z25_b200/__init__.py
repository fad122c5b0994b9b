"""B200-native GALA Louvain (PPoPP'25) — thin Python binding of libgala.so.

Argument marshalling only: every step of the method runs in the sm_100a CUDA
kernels behind the C ABI declared in include/gala.h.  There is no CPU
fallback: importing works without a GPU, but every call that needs the device
fails loudly if libgala.so or the GPU is missing.

    import paper_conf_ppopp_wangllwm00z25_b200 as gala
    g = gala.Graph.from_csr(row_ptr, col)           # numpy (host) or torch CUDA tensors
    g.run(gamma=1.0, tol=1e-6)
    labels, Q = g.communities(), g.modularity()
"""
from __future__ import annotations

import ctypes
import json
import os
import re

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# GALA_LIB_PATH: another in-tree build of the same library (tools/ab.py build-variant A/B only)
LIB_PATH = os.environ.get("GALA_LIB_PATH") or os.path.join(_HERE, "libgala.so")
HEADER_PATH = os.path.join(os.path.dirname(_HERE), "include", "gala.h")

STATUS = {0: "GALA_OK", 1: "GALA_E_INVALID", 2: "GALA_E_OVERFLOW", 3: "GALA_E_NOMEM", 4: "GALA_E_CUDA",
          5: "GALA_E_NCCL", 6: "GALA_E_STATE"}

_LIB = None


class GalaError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def lib():
    """Load libgala.so (raises if it was not built: there is no fallback path)."""
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} missing: build it with `make` or __graft_entry__.build()")
    L = ctypes.CDLL(LIB_PATH)
    i64, i32, u64, dbl, p, st = (ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_double,
                                 ctypes.c_void_p, ctypes.c_int)
    pp = ctypes.POINTER(ctypes.c_void_p)
    sig = {
        "gala_version": (ctypes.c_char_p, []),
        "gala_last_error": (ctypes.c_char_p, []),
        "gala_graph_from_csr": (st, [i64, p, p, p, ctypes.c_int, ctypes.c_size_t, pp]),
        "gala_graph_from_csr_device": (st, [i64, p, p, p, ctypes.c_int, ctypes.c_size_t, pp]),
        "gala_validate": (st, [p]),
        "gala_run": (st, [p, dbl, dbl, i32]),
        "gala_get_communities": (st, [p, p, i64, p]),
        "gala_get_communities_device": (st, [p, p, i64, p]),
        "gala_modularity": (st, [p, ctypes.POINTER(dbl)]),
        "gala_modularity_numerator": (st, [p, p, p, p, p, p]),
        "gala_graph_free": (None, [p]),
        "gala_set_option": (st, [p, ctypes.c_char_p, i64]),
        "gala_get_stats": (st, [p, p, i64, p]),
        "gala_get_trace_count": (st, [p, p]),
        "gala_get_trace_record": (st, [p, i64, p]),
        "gala_get_trace_labels": (st, [p, i64, p, i64]),
        "gala_get_kernel_stats": (st, [p, i32, ctypes.POINTER(ctypes.c_char_p), p, p, p, p]),
        "gala_nccl_unique_id": (st, [p]),
        "gala_loopback_unique_id": (st, [p]),
        "gala_graph_from_csr_dist": (st, [p, ctypes.c_int, ctypes.c_int, ctypes.c_int, i64, i64, i64, p, p, p,
                                          ctypes.c_size_t, pp]),
        "gala_partition_ranges": (st, [i64, p, ctypes.c_int, p]),
        "gala_set_allocator": (st, [p, p, p]),
        "gala_nmi_device": (st, [p, p, i64, ctypes.c_int, ctypes.c_size_t, ctypes.POINTER(dbl)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _LIB = L
    return L


def declared_functions() -> list[str]:
    """Names of every function declared in include/gala.h."""
    src = open(HEADER_PATH).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gala_[a-z0-9_]+)\s*\(", src)))


def _check(status: int):
    if status != 0:
        raise GalaError(status, lib().gala_last_error().decode(errors="replace"))


def _np_ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _i128(hi: int, lo: int) -> int:
    return (int(hi) << 64) | (int(lo) & 0xFFFFFFFFFFFFFFFF)


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_size_t, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_size_t, ctypes.c_void_p)
_ALLOC_HOOK = None   # keeps the ctypes callbacks alive while installed


def set_allocator(alloc=None, free=None):
    """Install a device allocator for every later library allocation (include/gala.h
    gala_set_allocator): alloc(bytes, device, stream) -> int pointer, free(ptr, bytes, device,
    stream).  set_allocator() restores the library's own stream-ordered pool."""
    global _ALLOC_HOOK
    if alloc is None and free is None:
        _check(lib().gala_set_allocator(None, None, None))
        _ALLOC_HOOK = None
        return

    def _a(nbytes, device, stream, ctx):
        try:
            return int(alloc(int(nbytes), int(device), int(stream)))
        except Exception:   # the library reports GALA_E_NOMEM
            return None

    def _f(ptr, nbytes, device, stream, ctx):
        free(int(ptr), int(nbytes), int(device), int(stream))

    hook = (ALLOC_FN(_a), FREE_FN(_f))
    _check(lib().gala_set_allocator(ctypes.cast(hook[0], ctypes.c_void_p), ctypes.cast(hook[1], ctypes.c_void_p),
                                    None))
    _ALLOC_HOOK = hook


def use_torch_allocator():
    """Route the library's device memory through torch.cuda's caching allocator
    (gala_set_allocator bound to caching_allocator_alloc / _delete)."""
    import torch

    def alloc(nbytes, device, stream):
        return torch.cuda.caching_allocator_alloc(nbytes, device, stream)

    def free(ptr, nbytes, device, stream):
        torch.cuda.caching_allocator_delete(ptr)

    set_allocator(alloc, free)


def version() -> str:
    return lib().gala_version().decode()


def partition_ranges(row_ptr: np.ndarray, world: int) -> np.ndarray:
    """Edge-balanced contiguous vertex ranges for `world` ranks (host-only helper of the C ABI)."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    out = np.zeros(world + 1, dtype=np.int64)
    _check(lib().gala_partition_ranges(len(rp) - 1, _np_ptr(rp), world, _np_ptr(out)))
    return out


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().gala_nccl_unique_id(buf))
    return buf.raw


def loopback_unique_id() -> bytes:
    """TEST HOOK: uid that runs the ranks of from_csr_dist as threads of one process on one GPU."""
    buf = ctypes.create_string_buffer(128)
    _check(lib().gala_loopback_unique_id(buf))
    return buf.raw


def nmi(x, y, stream: int = 0) -> float:
    """NMI of two partitions (include/gala.h gala_nmi_device, ref. [52]):
    x, y are int32 CUDA tensors of equal length with labels in [0, n).  Computed by the
    library's kernels on the tensors' device (argument marshalling only here)."""
    import torch
    if not (torch.is_tensor(x) and torch.is_tensor(y) and x.is_cuda and y.is_cuda):
        raise TypeError("nmi: x and y must be CUDA tensors")
    if x.dtype != torch.int32 or y.dtype != torch.int32 or x.numel() != y.numel() or x.device != y.device:
        raise ValueError("nmi: x and y must be int32 tensors of equal length on one device")
    xc, yc = x.contiguous(), y.contiguous()
    out = ctypes.c_double()
    _check(lib().gala_nmi_device(xc.data_ptr(), yc.data_ptr(), xc.numel(), x.device.index, stream,
                                 ctypes.byref(out)))
    return out.value


def local_rows(row_ptr, col, w, v0: int, v1: int):
    """Rows [v0, v1) of a CSR as (local_row_ptr, col, w) with global column ids (host arrays)."""
    rp = np.asarray(row_ptr, dtype=np.int64)
    a, b = int(rp[v0]), int(rp[v1])
    lrp = (rp[v0:v1 + 1] - a).astype(np.int64)
    lcol = np.ascontiguousarray(np.asarray(col, dtype=np.int32)[a:b])
    lw = None if w is None else np.ascontiguousarray(np.asarray(w, dtype=np.int64)[a:b])
    return lrp, lcol, lw


class Graph:
    """Handle of a graph resident on one GPU (or one rank's partition)."""

    def __init__(self, handle, n: int):
        self._h = handle
        self.n = int(n)

    # ------------------------------------------------------------ creation
    @classmethod
    def from_csr(cls, row_ptr, col, w=None, device: int = 0, stream: int = 0) -> "Graph":
        """Symmetric CSR: row_ptr int64[n+1], col int32[nnz], w int64[nnz] or None (all 1).

        numpy arrays (host) are copied host->device; torch CUDA tensors are copied device->device.
        """
        L = lib()
        h = ctypes.c_void_p()
        if hasattr(row_ptr, "is_cuda") and row_ptr.is_cuda:
            import torch
            rp = row_ptr.to(torch.int64).contiguous()
            cl = col.to(torch.int32).contiguous()
            ww = None if w is None else w.to(torch.int64).contiguous()
            n = rp.numel() - 1
            dev = rp.device.index if rp.device.index is not None else device
            _check(L.gala_graph_from_csr_device(n, rp.data_ptr(), cl.data_ptr(),
                                                None if ww is None else ww.data_ptr(), dev, stream,
                                                ctypes.byref(h)))
            return cls(h, n)
        if hasattr(row_ptr, "numpy"):
            row_ptr = row_ptr.numpy()
            col = col.numpy()
            w = None if w is None else w.numpy()
        rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
        cl = np.ascontiguousarray(col, dtype=np.int32)
        ww = None if w is None else np.ascontiguousarray(w, dtype=np.int64)
        n = len(rp) - 1
        _check(L.gala_graph_from_csr(n, _np_ptr(rp), _np_ptr(cl), _np_ptr(ww), device, stream,
                                     ctypes.byref(h)))
        return cls(h, n)

    @classmethod
    def from_graph(cls, g, device: int = 0, stream: int = 0) -> "Graph":
        """From a graphgen.CSR."""
        return cls.from_csr(g.row_ptr, g.col, g.w, device=device, stream=stream)

    @classmethod
    def from_csr_dist(cls, uid: bytes, rank: int, world: int, device: int, n_global: int, v_begin: int,
                      v_end: int, local_row_ptr, col, w=None, stream: int = 0) -> "Graph":
        rp = np.ascontiguousarray(local_row_ptr, dtype=np.int64)
        cl = np.ascontiguousarray(col, dtype=np.int32)
        ww = None if w is None else np.ascontiguousarray(w, dtype=np.int64)
        h = ctypes.c_void_p()
        ubuf = ctypes.create_string_buffer(uid, 128)
        _check(lib().gala_graph_from_csr_dist(ubuf, rank, world, device, n_global, v_begin, v_end, _np_ptr(rp),
                                              _np_ptr(cl), _np_ptr(ww), stream, ctypes.byref(h)))
        return cls(h, n_global)

    # ------------------------------------------------------------ run / results
    def set_option(self, key: str, value: int) -> "Graph":
        _check(lib().gala_set_option(self._h, key.encode(), int(value)))
        return self

    def validate(self):
        _check(lib().gala_validate(self._h))

    def run(self, gamma: float = 1.0, tol: float = 1e-6, max_levels: int = 0) -> "Graph":
        _check(lib().gala_run(self._h, float(gamma), float(tol), int(max_levels)))
        return self

    def communities(self) -> np.ndarray:
        out = np.zeros(self.n, dtype=np.int32)
        k = ctypes.c_int64()
        _check(lib().gala_get_communities(self._h, _np_ptr(out), self.n, ctypes.byref(k)))
        self.k = k.value
        return out

    def communities_device(self, out_tensor) -> int:
        k = ctypes.c_int64()
        _check(lib().gala_get_communities_device(self._h, out_tensor.data_ptr(), self.n, ctypes.byref(k)))
        return k.value

    def modularity(self) -> float:
        q = ctypes.c_double()
        _check(lib().gala_modularity(self._h, ctypes.byref(q)))
        return q.value

    def numerator(self):
        """(N, W, p, q): exact modularity numerator, Q = N / (q W^2)."""
        hi, lo, W, p, q = (ctypes.c_int64(), ctypes.c_uint64(), ctypes.c_int64(), ctypes.c_int64(),
                           ctypes.c_int64())
        _check(lib().gala_modularity_numerator(self._h, ctypes.byref(hi), ctypes.byref(lo), ctypes.byref(W),
                                               ctypes.byref(p), ctypes.byref(q)))
        return _i128(hi.value, lo.value), W.value, p.value, q.value

    def stats(self) -> dict:
        need = ctypes.c_int64()
        lib().gala_get_stats(self._h, None, 0, ctypes.byref(need))
        buf = ctypes.create_string_buffer(int(need.value) + 16)
        _check(lib().gala_get_stats(self._h, buf, len(buf), ctypes.byref(need)))
        return json.loads(buf.value.decode())

    def kernel_stats(self) -> dict:
        L = lib()
        cnt = ctypes.c_int32()
        L.gala_get_kernel_stats(self._h, -1, None, None, None, None, ctypes.byref(cnt))
        out = {}
        for k in range(cnt.value):
            name = ctypes.c_char_p()
            launches, ms, by = ctypes.c_int64(), ctypes.c_double(), ctypes.c_double()
            _check(L.gala_get_kernel_stats(self._h, k, ctypes.byref(name), ctypes.byref(launches), ctypes.byref(ms),
                                           ctypes.byref(by), ctypes.byref(cnt)))
            out[name.value.decode()] = dict(launches=launches.value, ms=ms.value, alg_bytes=by.value)
        return out

    def trace(self, labels: bool = False) -> list[dict]:
        L = lib()
        cnt = ctypes.c_int64()
        _check(L.gala_get_trace_count(self._h, ctypes.byref(cnt)))
        recs = []
        buf = np.zeros(16, dtype=np.int64)
        for i in range(cnt.value):
            _check(L.gala_get_trace_record(self._h, i, _np_ptr(buf)))
            r = dict(level=int(buf[0]), iter=int(buf[1]), n_level=int(buf[2]), n_active=int(buf[3]),
                     n_pruned=int(buf[4]), n_moved=int(buf[5]), N=_i128(buf[6], buf[7]),
                     edges_scanned=int(buf[8]), distinct=int(buf[9]), delta_used=int(buf[10]),
                     sync=int(buf[11]), n_fn=int(buf[12]), n_fp=int(buf[13]), us=int(buf[14]) / 1e3,
                     alg_bytes=int(buf[15]))
            if labels:
                lab = np.zeros(r["n_level"], dtype=np.int32)
                _check(L.gala_get_trace_labels(self._h, i, _np_ptr(lab), r["n_level"]))
                r["labels"] = lab
            recs.append(r)
        return recs

    def free(self):
        if self._h:
            lib().gala_graph_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.free()
