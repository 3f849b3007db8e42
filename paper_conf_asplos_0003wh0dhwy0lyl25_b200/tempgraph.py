"""Thin ctypes binding of include/tg.h (argument marshalling only).

Every step of the query path runs in libtempgraph.so's CUDA kernels; this module
only converts tensors/arrays to pointers.  There is no CPU fallback: if the
shared library is missing or no CUDA device is present, calls raise.

The functions keep the C names (tg_graph_create, tg_build_chains, tg_query, ...);
``Graph`` is a small convenience wrapper around them.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libtempgraph.so")

TG_OK, TG_ERR_INVALID, TG_ERR_RANGE, TG_ERR_NOMEM, TG_ERR_CUDA, TG_ERR_STATE, TG_ERR_NCCL = range(7)
TG_EAT, TG_LD, TG_FASTEST, TG_SHORTEST, TG_REACH, TG_LD_SOURCE = range(6)
PROBLEMS = {"eat": TG_EAT, "ld": TG_LD, "fp": TG_FASTEST, "fastest": TG_FASTEST,
            "sp": TG_SHORTEST, "shortest": TG_SHORTEST, "reach": TG_REACH, "lds": TG_LD_SOURCE}
TG_UNREACHED = 0xFFFFFFFF
TG_TMAX = 0x7FFFFFFE

EXPORTED = ["tg_graph_create", "tg_build_chains", "tg_query", "tg_graph_destroy", "tg_status_string",
            "tg_last_error", "tg_graph_info", "tg_export_chains", "tg_last_query_stats", "tg_set_option",
            "tg_kernel_launch_count", "tg_profile_enable", "tg_profile_report", "tg_release_cached_memory",
            "tg_nccl_unique_id", "tg_comm_create", "tg_comm_destroy", "tg_graph_attach_comm",
            "tg_query_topk", "tg_query_summary", "tg_graph_insert_edges", "tg_graph_create_streamed"]


class TGError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{_status_name(status)}: {msg}")
        self.status = status


class tg_window(ctypes.Structure):
    _fields_ = [("t_alpha", ctypes.c_uint32), ("t_omega", ctypes.c_uint32)]


class tg_info(ctypes.Structure):
    _fields_ = [("n_vertices", ctypes.c_uint32), ("n_edges", ctypes.c_uint64), ("n_nodes", ctypes.c_uint64),
                ("n_chains", ctypes.c_uint64), ("n_long_chains", ctypes.c_uint64),
                ("max_chain_len", ctypes.c_uint32), ("c_mirror", ctypes.c_uint32),
                ("device_bytes", ctypes.c_uint64), ("build_ms", ctypes.c_double), ("built", ctypes.c_int),
                ("n_chains_mirror", ctypes.c_uint64), ("host_bytes", ctypes.c_uint64), ("n_blocks", ctypes.c_uint32)]


class tg_query_stats(ctypes.Structure):
    _fields_ = [("rounds", ctypes.c_uint32), ("sub_batches", ctypes.c_uint32),
                ("slots_relaxed", ctypes.c_uint64), ("kernel_launches", ctypes.c_uint64),
                ("slots_union", ctypes.c_uint64)]


_lib = None


def load_library(path: str = LIB_PATH):
    """Load libtempgraph.so (raises if it has not been built: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"libtempgraph.so not built ({path}); run __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    P, u32, u64, i64 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64
    st = ctypes.c_int
    lib.tg_graph_create.restype = st
    lib.tg_graph_create.argtypes = [u32, u64, P, P, P, P, P, ctypes.c_int, ctypes.POINTER(P)]
    lib.tg_build_chains.restype = st
    lib.tg_build_chains.argtypes = [P]
    lib.tg_query.restype = st
    lib.tg_query.argtypes = [P, ctypes.c_int, P, u32, tg_window, P, P, P]
    lib.tg_graph_create_streamed.restype = st
    lib.tg_graph_create_streamed.argtypes = [u32, u64, P, P, P, P, P, ctypes.c_int, u64, ctypes.POINTER(P)]
    lib.tg_graph_insert_edges.restype = st
    lib.tg_graph_insert_edges.argtypes = [P, u64, P, P, P, P, P]
    lib.tg_query_topk.restype = st
    lib.tg_query_topk.argtypes = [P, ctypes.c_int, P, u32, tg_window, u32, P, P, P]
    lib.tg_query_summary.restype = st
    lib.tg_query_summary.argtypes = [P, ctypes.c_int, P, u32, tg_window, P, P, P]
    lib.tg_graph_destroy.restype = None
    lib.tg_graph_destroy.argtypes = [P]
    lib.tg_status_string.restype = ctypes.c_char_p
    lib.tg_status_string.argtypes = [ctypes.c_int]
    lib.tg_last_error.restype = ctypes.c_char_p
    lib.tg_last_error.argtypes = []
    lib.tg_graph_info.restype = st
    lib.tg_graph_info.argtypes = [P, ctypes.POINTER(tg_info)]
    lib.tg_export_chains.restype = st
    lib.tg_export_chains.argtypes = [P, ctypes.c_int, P, P, P, P, P, P]
    lib.tg_last_query_stats.restype = st
    lib.tg_last_query_stats.argtypes = [P, ctypes.POINTER(tg_query_stats), P]
    lib.tg_set_option.restype = st
    lib.tg_set_option.argtypes = [P, ctypes.c_char_p, i64]
    lib.tg_kernel_launch_count.restype = u64
    lib.tg_kernel_launch_count.argtypes = []
    lib.tg_nccl_unique_id.restype = st
    lib.tg_nccl_unique_id.argtypes = [P]
    lib.tg_comm_create.restype = st
    lib.tg_comm_create.argtypes = [P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(P)]
    lib.tg_comm_destroy.restype = None
    lib.tg_comm_destroy.argtypes = [P]
    lib.tg_graph_attach_comm.restype = st
    lib.tg_graph_attach_comm.argtypes = [P, P, ctypes.c_int]
    lib.tg_release_cached_memory.restype = None
    lib.tg_release_cached_memory.argtypes = []
    lib.tg_profile_enable.restype = None
    lib.tg_profile_enable.argtypes = [ctypes.c_int]
    lib.tg_profile_report.restype = ctypes.c_int
    lib.tg_profile_report.argtypes = [ctypes.c_char_p, u64]
    _lib = lib
    return lib


def _status_name(s):
    try:
        return load_library().tg_status_string(s).decode()
    except Exception:
        return f"status {s}"


def _check(status):
    if status != TG_OK:
        raise TGError(status, load_library().tg_last_error().decode())


def _ptr(x):
    """Pointer of a torch tensor (CPU or CUDA) or numpy array; None -> NULL."""
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        assert x.flags["C_CONTIGUOUS"] and x.itemsize == 4
        return x.ctypes.data
    # torch tensor
    assert x.is_contiguous() and x.element_size() == 4, "expected contiguous 32-bit tensor"
    return x.data_ptr()


# --------------------------------------------------------------------------- C names
def tg_graph_create(n_vertices, u, v, t_start, duration, weight=None, device=0):
    lib = load_library()
    h = ctypes.c_void_p()
    m = int(u.shape[0])
    _check(lib.tg_graph_create(int(n_vertices), m, _ptr(u), _ptr(v), _ptr(t_start), _ptr(duration), _ptr(weight),
                               int(device), ctypes.byref(h)))
    return h


def tg_graph_insert_edges(g, u, v, t_start, duration, weight=None):
    _check(load_library().tg_graph_insert_edges(g, int(u.shape[0]), _ptr(u), _ptr(v), _ptr(t_start), _ptr(duration),
                                                _ptr(weight)))


def tg_graph_create_streamed(n_vertices, u, v, t_start, duration, weight=None, device=0, block_edges=1 << 26):
    """Out-of-memory graph (host arrays only; see include/tg.h)."""
    lib = load_library()
    h = ctypes.c_void_p()
    m = int(u.shape[0])
    _check(lib.tg_graph_create_streamed(int(n_vertices), m, _ptr(u), _ptr(v), _ptr(t_start), _ptr(duration),
                                        _ptr(weight), int(device), int(block_edges), ctypes.byref(h)))
    return h


def tg_build_chains(g):
    _check(load_library().tg_build_chains(g))


def tg_query(g, problem, sources, window, out, pred=None, stream=None):
    lib = load_library()
    src = np.ascontiguousarray(np.asarray(sources, dtype=np.uint32))
    w = tg_window(int(window[0]), int(window[1]))
    s = None
    if stream is not None:
        s = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
    _check(lib.tg_query(g, int(problem), src.ctypes.data, int(src.shape[0]), w, _ptr(out), _ptr(pred), s))


def tg_query_topk(g, problem, sources, window, K, out_vertex, out_value, stream=None):
    lib = load_library()
    src = np.ascontiguousarray(np.asarray(sources, dtype=np.uint32))
    w = tg_window(int(window[0]), int(window[1]))
    s = None if stream is None else (stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))
    _check(lib.tg_query_topk(g, int(problem), src.ctypes.data, int(src.shape[0]), w, int(K), _ptr(out_vertex),
                             _ptr(out_value), s))


def tg_query_summary(g, problem, sources, window, stream=None):
    """Returns (count uint64[k], sum uint64[k]) host arrays."""
    lib = load_library()
    src = np.ascontiguousarray(np.asarray(sources, dtype=np.uint32))
    w = tg_window(int(window[0]), int(window[1]))
    cnt = np.zeros(len(src), np.uint64)
    sm = np.zeros(len(src), np.uint64)
    s = None if stream is None else (stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))
    _check(lib.tg_query_summary(g, int(problem), src.ctypes.data, int(src.shape[0]), w, cnt.ctypes.data,
                                sm.ctypes.data, s))
    return cnt, sm


def tg_graph_destroy(g):
    load_library().tg_graph_destroy(g)


def tg_graph_info(g) -> dict:
    info = tg_info()
    _check(load_library().tg_graph_info(g, ctypes.byref(info)))
    return {k: getattr(info, k) for k, _ in tg_info._fields_}


def tg_export_chains(g, m, n_chains, mirrored=False, shortcuts=True):
    off = np.empty(n_chains + 1, np.uint64)
    edges = np.empty(max(m, 1), np.uint32)
    sc = {k: np.empty(max(n_chains, 1), np.uint32) for k in ("tail_v", "arr", "elapsed")}
    sw = np.empty(max(n_chains, 1), np.uint64)
    args = [sc["tail_v"].ctypes.data, sc["arr"].ctypes.data, sw.ctypes.data, sc["elapsed"].ctypes.data] \
        if shortcuts else [None] * 4
    _check(load_library().tg_export_chains(g, int(mirrored), off.ctypes.data, edges.ctypes.data, *args))
    res = {"chain_off": off.astype(np.int64), "chain_edges": edges[:m]}
    if shortcuts:
        res.update({k: a[:n_chains] for k, a in sc.items()})
        res["sum_w"] = sw[:n_chains]
    return res


def tg_last_query_stats(g, n_queries=0):
    st = tg_query_stats()
    per = np.zeros(max(n_queries, 1), np.uint64)
    _check(load_library().tg_last_query_stats(g, ctypes.byref(st), per.ctypes.data if n_queries else None))
    d = {k: getattr(st, k) for k, _ in tg_query_stats._fields_}
    if n_queries:
        d["per_query_relax"] = per[:n_queries]
    return d


def tg_set_option(g, key: str, value: int):
    _check(load_library().tg_set_option(g, key.encode(), int(value)))


def tg_kernel_launch_count() -> int:
    return int(load_library().tg_kernel_launch_count())


def tg_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(load_library().tg_nccl_unique_id(buf))
    return buf.raw


def tg_comm_create(unique_id: bytes, rank: int, world: int, device: int):
    h = ctypes.c_void_p()
    buf = ctypes.create_string_buffer(bytes(unique_id), 128)
    _check(load_library().tg_comm_create(buf, int(rank), int(world), int(device), ctypes.byref(h)))
    return h


def tg_comm_destroy(c):
    load_library().tg_comm_destroy(c)


def tg_graph_attach_comm(g, c, mode: int):
    _check(load_library().tg_graph_attach_comm(g, c, int(mode)))


def tg_release_cached_memory():
    load_library().tg_release_cached_memory()


def tg_profile_enable(on=True):
    """True / 1: every kernel; 2: only the EAT-family relaxation kernels; False / 0: off."""
    load_library().tg_profile_enable(int(on) if not isinstance(on, bool) else (1 if on else 0))


def tg_profile_report() -> dict:
    """{kernel: (launches, total_ms)} of the launches recorded since the last report."""
    import json
    lib = load_library()
    need = lib.tg_profile_report(None, 0)
    buf = ctypes.create_string_buffer(max(need, 2) + 4096)
    lib.tg_profile_report(buf, len(buf))
    return {k: (int(v[0]), float(v[1])) for k, v in json.loads(buf.value.decode()).items()}


# --------------------------------------------------------------------------- convenience
class Graph:
    """Owning wrapper: Graph(n, u, v, t, dur, w=None, device=0).build().query(...)."""

    def __init__(self, n, u, v, t, dur, w=None, device=0, block_edges=None):
        """block_edges: None = device-resident graph; else an out-of-memory graph
        streamed in time blocks of at most that many edges (host arrays)."""
        self.n = int(n)
        self.m = int(u.shape[0])
        self.device = device
        if block_edges is None:
            self.h = tg_graph_create(n, u, v, t, dur, w, device)
        else:
            self.h = tg_graph_create_streamed(n, u, v, t, dur, w, device, block_edges)

    def build(self):
        tg_build_chains(self.h)
        return self

    def insert_edges(self, u, v, t, dur, w=None):
        tg_graph_insert_edges(self.h, u, v, t, dur, w)
        self.m += int(u.shape[0])
        return self

    def info(self):
        return tg_graph_info(self.h)

    def set_option(self, key, value):
        tg_set_option(self.h, key, value)
        return self

    def query(self, problem, sources, window=(0, TG_TMAX), with_pred=False, out=None, pred=None, stream=None):
        """Returns torch.int32 CUDA tensors [k, n] holding uint32 bits (out[, pred])."""
        import torch
        p = PROBLEMS[problem] if isinstance(problem, str) else int(problem)
        k = len(sources)
        dev = torch.device("cuda", self.device)
        if out is None:
            out = torch.empty((k, self.n), dtype=torch.int32, device=dev)
        if with_pred and pred is None:
            pred = torch.empty((k, self.n), dtype=torch.int32, device=dev)
        tg_query(self.h, p, sources, window, out, pred, stream)
        return (out, pred) if with_pred else out

    def topk(self, problem, sources, K, window=(0, TG_TMAX)):
        """(vertices, values): torch.int32 CUDA tensors [k, K] (uint32 bits)."""
        import torch
        p = PROBLEMS[problem] if isinstance(problem, str) else int(problem)
        dev = torch.device("cuda", self.device)
        ov = torch.empty((len(sources), K), dtype=torch.int32, device=dev)
        oval = torch.empty((len(sources), K), dtype=torch.int32, device=dev)
        tg_query_topk(self.h, p, sources, window, K, ov, oval)
        return ov, oval

    def summary(self, problem, sources, window=(0, TG_TMAX)):
        p = PROBLEMS[problem] if isinstance(problem, str) else int(problem)
        return tg_query_summary(self.h, p, sources, window)

    def export_chains(self, mirrored=False, shortcuts=True):
        info = self.info()
        nc = info["n_chains_mirror" if mirrored else "n_chains"]
        return tg_export_chains(self.h, self.m, nc, mirrored, shortcuts)

    def last_stats(self, n_queries=0):
        return tg_last_query_stats(self.h, n_queries)

    def close(self):
        if self.h:
            tg_graph_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def as_u32(x) -> np.ndarray:
    """uint32 numpy view of a torch int32 tensor / array (bits unchanged)."""
    if hasattr(x, "detach"):
        x = x.detach().cpu().numpy()
    return np.ascontiguousarray(x).view(np.uint32)
