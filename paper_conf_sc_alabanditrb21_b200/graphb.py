"""Thin Python binding of the C ABI (include/graphb.h): argument marshalling
only.  Every step of the balancing path runs in libgraphb.so's sm_100a
kernels; if the library or a CUDA device is missing, calls raise -- there is
no CPU fallback.

Names follow the C ABI: load_csr, balance, free, balance_range, tree_debug,
balance_given_tree.  ``balance`` additionally shards trees over the ranks of
an initialised torch.distributed process group (tree t -> rank t mod W,
PAPER.md L248) and all-reduces the integer counters (one NCCL all-reduce).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

GB_OK, GB_EINVAL, GB_ESTATE, GB_ENOMEM, GB_ECUDA = 0, -1, -2, -3, -4
PHASES = ("init", "bfs", "bottom_up", "top_down", "cycles", "accumulate")
_ERRNAMES = {GB_EINVAL: "GB_EINVAL", GB_ESTATE: "GB_ESTATE", GB_ENOMEM: "GB_ENOMEM",
             GB_ECUDA: "GB_ECUDA"}


class GraphBError(RuntimeError):
    def __init__(self, rc, msg):
        super().__init__(f"{_ERRNAMES.get(rc, rc)}: {msg}")
        self.rc = rc


_lib = None


def library_path() -> str:
    return _build.LIB


def lib():
    """Load libgraphb.so (built in-tree by __graft_entry__.build())."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("GRAPHB_LIB", _build.LIB)   # alternative in-tree builds (experiments)
    if not os.path.exists(path):
        raise RuntimeError(f"{path} is missing: run __graft_entry__.build() "
                           "(the CUDA library is required; there is no fallback)")
    L = ctypes.CDLL(path)
    P, i64, u64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_int
    sig = {
        "gb_load_csr": (i32, [i64, i64, P, P, P]),
        "gb_balance": (i32, [i64, u64, P, P]),
        "gb_free": (None, []),
        "gb_balance_range": (i32, [i64, i64, i64, u64, P, P, P]),
        "gb_tree_debug": (i32, [i64, u64, P, P, P, P, P, P, P]),
        "gb_balance_given_tree": (i32, [P, P, P, P]),
        "gb_set_option": (i32, [ctypes.c_char_p, i64]),
        "gb_get_stats": (i32, [P, i32, P, i32]),
        "gb_tree_stats": (i64, [P, P, i64]),
        "gb_cloud_states": (i64, [P, P, i64]),
        "gb_msbfs_profile": (i32, [P]),
        "gb_label_profile": (i32, [P]),
        "gb_graph_info": (i32, [P, P, P]),
        "gb_graph_debug": (i32, [P, P, P, P, P]),
        "gb_selftest": (i32, []),
        "gb_last_error": (ctypes.c_char_p, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def exported_symbols():
    return ["gb_load_csr", "gb_balance", "gb_free", "gb_balance_range", "gb_tree_debug",
            "gb_balance_given_tree", "gb_set_option", "gb_get_stats", "gb_tree_stats",
            "gb_graph_info", "gb_graph_debug", "gb_selftest", "gb_last_error", "gb_msbfs_profile",
            "gb_label_profile", "gb_cloud_states"]


def _check(rc):
    if rc != GB_OK:
        raise GraphBError(rc, lib().gb_last_error().decode())
    return rc


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def last_error() -> str:
    return lib().gb_last_error().decode()


def selftest():
    return _check(lib().gb_selftest())


def load_csr(row_ptr, col_idx, sign):
    """gb_load_csr: host arrays (int64 row_ptr[n+1], int32 col[2m], int8 sign[2m])."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    sign = np.ascontiguousarray(sign, dtype=np.int8)
    n = len(row_ptr) - 1
    m = len(col_idx) // 2
    if len(col_idx) != 2 * m or len(sign) != len(col_idx):
        raise GraphBError(GB_EINVAL, "col/sign must have the same even length")
    _check(lib().gb_load_csr(n, m, _ptr(row_ptr), _ptr(col_idx) if m else None,
                             _ptr(sign) if m else None))
    return n, m


def load_graph(g):
    """Load a graphgen.SignedCSR-like object (row_ptr, col, sign)."""
    return load_csr(g.row_ptr, g.col, g.sign)


def free():
    lib().gb_free()


def graph_info():
    n, m, c = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    _check(lib().gb_graph_info(ctypes.byref(n), ctypes.byref(m), ctypes.byref(c)))
    return n.value, m.value, c.value


def graph_debug(edges=True, slot_eid=True, comp=True):
    """Ingest results (a.1): edge table by eid, eid of every slot, components
    (arrays not asked for come back as None)."""
    n, m, _ = graph_info()
    eu = np.zeros(max(m, 1), np.int32) if edges else None
    ev = np.zeros(max(m, 1), np.int32) if edges else None
    en = np.zeros(max(m, 1), np.int8) if edges else None
    se = np.zeros(max(2 * m, 1), np.uint32) if slot_eid else None
    cp = np.zeros(n, np.int32) if comp else None
    _check(lib().gb_graph_debug(_ptr(eu), _ptr(ev), _ptr(en), _ptr(se), _ptr(cp)))
    cut = lambda a, k: a[:k] if a is not None else None
    return cut(eu, m), cut(ev, m), cut(en, m), cut(se, 2 * m), cp


def set_option(key: str, value: int):
    _check(lib().gb_set_option(key.encode(), int(value)))


def balance_host(num_trees, seed, out=None):
    """gb_balance with host outputs: (edge_flip_counts uint32[m], vertex_agree uint32[n]).
    `out` = optional caller arrays (uint32, >= max(m,1) and n long; e.g. pinned)."""
    n, m, _ = graph_info()
    if out is not None:
        cnt, agree = out
        if cnt.dtype != np.uint32 or agree.dtype != np.uint32 or len(cnt) < max(m, 1) or len(agree) < n:
            raise GraphBError(GB_EINVAL, "out arrays must be uint32 of length >= m and n")
    else:
        cnt = np.zeros(max(m, 1), np.uint32)
        agree = np.zeros(n, np.uint32)
    _check(lib().gb_balance(int(num_trees), int(seed) & (2**64 - 1), _ptr(cnt), _ptr(agree)))
    return cnt[:m], agree


def balance_range(t_begin, t_end, t_stride, seed, d_edge_cnt, d_vertex_agree, stream=None):
    """gb_balance_range into int32 CUDA tensors (accumulating)."""
    import torch
    for t in (d_edge_cnt, d_vertex_agree):
        if not (t.is_cuda and t.dtype == torch.int32 and t.is_contiguous()):
            raise GraphBError(GB_EINVAL, "outputs must be contiguous int32 CUDA tensors")
    s = stream.cuda_stream if stream is not None else torch.cuda.current_stream().cuda_stream
    if s == 0:
        s = 1   # torch's legacy default stream: cudaStreamLegacy (NULL would mean the library's own stream)
    _check(lib().gb_balance_range(int(t_begin), int(t_end), int(t_stride), int(seed) & (2**64 - 1),
                                  ctypes.c_void_p(d_edge_cnt.data_ptr()),
                                  ctypes.c_void_p(d_vertex_agree.data_ptr()), ctypes.c_void_p(s)))


def balance(num_trees, seed, group=None):
    """The frustration cloud over trees 0..num_trees-1 (Alg. 2): host numpy
    arrays (edge_flip_counts uint32[m], vertex_agree uint32[n]).

    Without an initialised torch.distributed group this is gb_balance.  With
    one, rank r balances trees {t : t mod W == r} into one int32 device buffer
    [cnt | agree] and one all-reduce(SUM) merges the shards;
    every rank returns the same arrays, of the same type as without a group.
    """
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return balance_host(num_trees, seed)
    _, m, _ = graph_info()
    cnt, agree = sharded_balance(num_trees, seed, dist.get_rank(group), dist.get_world_size(group),
                                 _device_range, m, group=group)
    return (cnt.cpu().numpy().astype(np.uint32), agree.cpu().numpy().astype(np.uint32))


def counter_buffer(device=None):
    """One int32 device buffer [edge counters (m) | vertex agree (n)]: the
    layout of the all-reduce, so no concatenation is needed per call."""
    import torch
    n, m, _ = graph_info()
    dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
    return torch.zeros(m + n, dtype=torch.int32, device=dev)


def balance_range_buf(t_begin, t_end, t_stride, seed, buf, stream=None):
    """gb_balance_range into a counter_buffer() (accumulating)."""
    _, m, _ = graph_info()
    balance_range(t_begin, t_end, t_stride, seed, buf[:m], buf[m:], stream)


def _device_range(t_begin, t_end, stride, seed):
    buf = counter_buffer()
    balance_range_buf(t_begin, t_end, stride, seed, buf)
    return buf


def sharded_balance(num_trees, seed, rank, world, range_fn, m, group=None):
    """Host logic of the multi-GPU path, independent of the
    backend: rank computes its tree shard with range_fn(t_begin, t_end,
    stride, seed) -> one int32 tensor [cnt (m) | agree (n)], then one
    all_reduce(SUM) of that buffer in place.  Returns (cnt, agree) views."""
    import torch.distributed as dist
    buf = range_fn(rank, num_trees, world, seed)
    dist.all_reduce(buf, op=dist.ReduceOp.SUM, group=group)
    return buf[:m], buf[m:]


def tree_debug(t, seed):
    """Every stage of one tree (gb_tree_debug) as a dict of numpy arrays."""
    n, m, _ = graph_info()
    out = {k: np.zeros(n, np.int32) for k in ("parent", "dist", "pre", "size")}
    flip = np.zeros(max(m, 1), np.uint8)
    sk = ctypes.c_uint64()
    nc = ctypes.c_int64()
    _check(lib().gb_tree_debug(int(t), int(seed) & (2**64 - 1), _ptr(out["parent"]), _ptr(out["dist"]),
                               _ptr(out["pre"]), _ptr(out["size"]), _ptr(flip), ctypes.byref(sk),
                               ctypes.byref(nc)))
    out["flip"] = flip[:m]
    out["sum_cycle_len"] = sk.value
    out["num_cycles"] = nc.value
    return out


def balance_given_tree(parent):
    """Alg. 3 on a caller tree: (flip uint8[m], sum_cycle_len, num_cycles)."""
    parent = np.ascontiguousarray(parent, dtype=np.int32)
    n, m, _ = graph_info()
    flip = np.zeros(max(m, 1), np.uint8)
    sk = ctypes.c_uint64()
    nc = ctypes.c_int64()
    _check(lib().gb_balance_given_tree(_ptr(parent), _ptr(flip), ctypes.byref(sk), ctypes.byref(nc)))
    return flip[:m], sk.value, nc.value


def stats():
    ints = np.zeros(11, np.int64)
    ph = np.zeros(len(PHASES), np.float64)
    lib().gb_get_stats(_ptr(ints), 11, _ptr(ph), len(PHASES))
    keys = ("trees", "sum_cycle_len", "cycles", "launches", "batches", "max_depth", "batch",
            "cycle_group", "harary_violations", "sub", "bfs_group")
    d = {k: int(v) for k, v in zip(keys, ints)}
    d["phase_ms"] = {k: float(v) for k, v in zip(PHASES, ph)}
    return d


def tree_stats(max_trees=1 << 16):
    """Per-tree (sum of cycle lengths, cycles, depth, state signature) of the
    last balance call."""
    out = np.zeros(4 * max_trees, np.uint64)
    ids = np.zeros(max_trees, np.int64)
    k = lib().gb_tree_stats(_ptr(out), _ptr(ids), max_trees)
    return ids[:k], out[: 4 * k].reshape(k, 4)


def cloud_states(max_states=1 << 16):
    """Frustration-cloud analytics of the last balance call (SURVEY §8 f.2,
    gb_cloud_states, counted on the device): {state signature: number of
    sampled trees reaching that nearest balanced state}.  len() of it is the
    number of distinct states found."""
    sig = np.zeros(max_states, np.uint64)
    cnt = np.zeros(max_states, np.uint64)
    k = lib().gb_cloud_states(_ptr(sig), _ptr(cnt), max_states)
    if k < 0:
        _check(int(k))
    k = min(int(k), max_states)
    return {int(s): int(c) for s, c in zip(sig[:k], cnt[:k])}


def msbfs_profile():
    """Per-level BFS phase times (ms) of the last batch: list of
    (level, discovery, parents, hubs) -- needs set_option("msprof", 1)."""
    out = np.zeros(1024, dtype=np.uint64)
    _check(lib().gb_msbfs_profile(_ptr(out)))
    t = out.reshape(256, 4).astype(np.int64)
    rows = []
    for L in range(256):
        if t[L, 0] == 0:
            break
        nxt = t[L + 1, 0] if L + 1 < 256 and t[L + 1, 0] else t[L, 3]
        rows.append((L, (t[L, 1] - t[L, 0]) / 1e6, (t[L, 2] - t[L, 1]) / 1e6, (nxt - t[L, 2]) / 1e6))
    return rows


def label_profile():
    """Per-level Alg. 4 times (ms) of the last labelling launch: list of
    (level, vertices, bottom-up ms, top-down ms) -- needs set_option("msprof", 1)."""
    out = np.zeros(1024, dtype=np.uint64)
    _check(lib().gb_label_profile(_ptr(out)))
    t = out.reshape(256, 4).astype(np.int64)
    D = int(np.max(np.nonzero(t[:, 1])[0])) - 1 if t[:, 1].any() else -1
    rows = []
    for L in range(D + 1):
        bu = (t[L - 1, 0] - t[L, 0]) / 1e6 if L >= 1 and t[L, 0] else 0.0   # bottom-up runs D..1
        td = (t[L + 1, 1] - t[L, 1]) / 1e6
        rows.append((L, int(t[L, 2]), bu, td))
    return rows
