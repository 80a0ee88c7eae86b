"""TEST INFRASTRUCTURE ONLY: ctypes wrapper of the plain C oracle (oracle.c).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product (``paper_conf_sc_alabanditrb21_b200``) never imports it and shares no
code with it.  See oracle.h for the PAPER.md passage behind each function.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_HDR = os.path.join(_HERE, "oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")

OR_OK, OR_EINVAL, OR_ENOMEM, OR_EUNBAL = 0, -1, -3, -5


def build(force: bool = False) -> str:
    """Compile liboracle.so with plain gcc -O2 (single-threaded C99)."""
    stale = (not os.path.exists(_LIB)) or any(
        os.path.getmtime(p) > os.path.getmtime(_LIB) for p in (_SRC, _HDR))
    if force or stale:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-Wall", "-shared", "-fPIC",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        i64, u64 = ctypes.c_int64, ctypes.c_uint64
        L.or_mix64.restype = u64; L.or_mix64.argtypes = [u64]
        L.or_splitmix64_next.restype = u64; L.or_splitmix64_next.argtypes = [ctypes.POINTER(u64)]
        L.or_tkey.restype = u64; L.or_tkey.argtypes = [u64, i64]
        L.or_rkey.restype = u64; L.or_rkey.argtypes = [u64, i64, i64]
        L.or_pscore.restype = ctypes.c_uint32
        L.or_pscore.argtypes = [u64, i64, ctypes.c_int32, ctypes.c_int32]
        L.or_build.restype = ctypes.c_int
        L.or_build.argtypes = [i64, i64, P, P, P, ctypes.POINTER(P)]
        L.or_free.restype = None; L.or_free.argtypes = [P]
        for f in ("or_n", "or_m", "or_ncomp"):
            getattr(L, f).restype = i64; getattr(L, f).argtypes = [P]
        L.or_edges.restype = None; L.or_edges.argtypes = [P, P, P, P]
        L.or_components.restype = None; L.or_components.argtypes = [P, P, P, P]
        L.or_bfs_tree.restype = ctypes.c_int; L.or_bfs_tree.argtypes = [P, u64, i64, P, P, P]
        L.or_balance_tree.restype = ctypes.c_int
        L.or_balance_tree.argtypes = [P, P, P, ctypes.POINTER(u64), ctypes.POINTER(i64),
                                      ctypes.POINTER(ctypes.c_int32)]
        L.or_preorder.restype = ctypes.c_int; L.or_preorder.argtypes = [P, P, P, P]
        L.or_harary.restype = ctypes.c_int; L.or_harary.argtypes = [P, P, P, P]
        L.or_state_signature.restype = u64
        L.or_state_signature.argtypes = [P, i64]
        L.or_balance.restype = ctypes.c_int
        L.or_balance.argtypes = [P, i64, i64, i64, u64, P, P, P]
        L.or_balance_m.restype = ctypes.c_int
        L.or_balance_m.argtypes = [P, i64, i64, i64, u64, ctypes.c_int, P, P, P]
        L.or_wdraw.restype = u64; L.or_wdraw.argtypes = [u64, i64, ctypes.c_int32, ctypes.c_uint32]
        L.or_dstart.restype = u64; L.or_dstart.argtypes = [u64, i64, ctypes.c_int32]
        L.or_dfs_tree.restype = ctypes.c_int
        L.or_dfs_tree.argtypes = [P, u64, i64, P]
        L.or_wilson_tree.restype = ctypes.c_int
        L.or_wilson_tree.argtypes = [P, u64, i64, ctypes.c_int, P, P]
        _lib = L
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def mix64(z):
    return int(lib().or_mix64(ctypes.c_uint64(z & (2**64 - 1))))


def splitmix64_stream(state, k):
    s = ctypes.c_uint64(state)
    return [int(lib().or_splitmix64_next(ctypes.byref(s))) for _ in range(k)]


def tkey(seed, t):
    return int(lib().or_tkey(seed, t))


def rkey(seed, t, c):
    return int(lib().or_rkey(seed, t, c))


def pscore(seed, t, a, b):
    return int(lib().or_pscore(seed, t, a, b))


def wdraw(seed, t, u, j):
    return int(lib().or_wdraw(seed & (2**64 - 1), t, u, j))


def dstart(seed, t, u):
    return int(lib().or_dstart(seed & (2**64 - 1), t, u))


def state_signature(flip):
    flip = np.ascontiguousarray(flip, dtype=np.uint8)
    return int(lib().or_state_signature(_p(flip) if len(flip) else None, len(flip)))


class OracleError(RuntimeError):
    def __init__(self, rc, what):
        super().__init__(f"oracle {what} failed with code {rc}")
        self.rc = rc


class Graph:
    """An oracle-side copy of a signed CSR graph (validated like gb_load_csr)."""

    def __init__(self, row_ptr, col, sign):
        L = lib()
        self.row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
        self.col = np.ascontiguousarray(col, dtype=np.int32)
        self.sign = np.ascontiguousarray(sign, dtype=np.int8)
        n = len(self.row_ptr) - 1
        m = len(self.col) // 2
        h = ctypes.c_void_p()
        rc = L.or_build(n, m, _p(self.row_ptr), _p(self.col), _p(self.sign), ctypes.byref(h))
        if rc != OR_OK:
            raise OracleError(rc, "or_build")
        self._h = h
        self.n, self.m = n, m
        self.ncomp = int(L.or_ncomp(h))

    @classmethod
    def from_csr(cls, g):
        return cls(g.row_ptr, g.col, g.sign)

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and _lib is not None:
            _lib.or_free(h)
            self._h = None

    def edges(self):
        u = np.zeros(self.m, np.int32); v = np.zeros(self.m, np.int32); neg = np.zeros(self.m, np.int8)
        lib().or_edges(self._h, _p(u), _p(v), _p(neg))
        return u, v, neg

    def components(self):
        comp = np.zeros(self.n, np.int32); coff = np.zeros(self.ncomp + 1, np.int64)
        cverts = np.zeros(self.n, np.int32)
        lib().or_components(self._h, _p(comp), _p(coff), _p(cverts))
        return comp, coff, cverts

    def bfs_tree(self, seed, t):
        parent = np.zeros(self.n, np.int32); dist = np.zeros(self.n, np.int32)
        peid = np.zeros(self.n, np.int32)
        rc = lib().or_bfs_tree(self._h, seed, t, _p(parent), _p(dist), _p(peid))
        if rc != OR_OK:
            raise OracleError(rc, "or_bfs_tree")
        return parent, dist, peid

    def balance_tree(self, parent):
        parent = np.ascontiguousarray(parent, dtype=np.int32)
        flip = np.zeros(max(self.m, 1), np.uint8)
        sk = ctypes.c_uint64(); nc = ctypes.c_int64(); md = ctypes.c_int32()
        rc = lib().or_balance_tree(self._h, _p(parent), _p(flip), ctypes.byref(sk),
                                   ctypes.byref(nc), ctypes.byref(md))
        if rc != OR_OK:
            raise OracleError(rc, "or_balance_tree")
        return flip[: self.m], int(sk.value), int(nc.value), int(md.value)

    def preorder(self, parent):
        parent = np.ascontiguousarray(parent, dtype=np.int32)
        pre = np.zeros(self.n, np.int32); size = np.zeros(self.n, np.int32)
        rc = lib().or_preorder(self._h, _p(parent), _p(pre), _p(size))
        if rc != OR_OK:
            raise OracleError(rc, "or_preorder")
        return pre, size

    def harary(self, flip):
        flip = np.ascontiguousarray(flip, dtype=np.uint8)
        if len(flip) == 0:
            flip = np.zeros(1, np.uint8)
        side = np.zeros(self.n, np.uint8); d2 = np.zeros(self.n, np.uint8)
        rc = lib().or_harary(self._h, _p(flip), _p(side), _p(d2))
        if rc != OR_OK:
            raise OracleError(rc, "or_harary")
        return side, d2

    def wilson_tree(self, seed, t, order=0):
        """Uniform spanning forest (Wilson, reading R17): (parent, pops)."""
        parent = np.zeros(self.n, np.int32); pops = np.zeros(self.n, np.uint32)
        rc = lib().or_wilson_tree(self._h, seed, t, order, _p(parent), _p(pops))
        if rc != OR_OK:
            raise OracleError(rc, "or_wilson_tree")
        return parent, pops

    def dfs_tree(self, seed, t):
        """Random-start DFS tree (reading R18): parent (-1 at the roots)."""
        parent = np.zeros(self.n, np.int32)
        rc = lib().or_dfs_tree(self._h, seed, t, _p(parent))
        if rc != OR_OK:
            raise OracleError(rc, "or_dfs_tree")
        return parent

    def balance(self, num_trees, seed, t_begin=0, stride=1, with_stats=False, sampler=0):
        """Frustration cloud over trees t_begin, t_begin+stride, ... < num_trees
        (sampler 0 = BFS trees, 1 = uniform spanning trees, 2 = DFS trees)."""
        cnt = np.zeros(max(self.m, 1), np.uint32); agree = np.zeros(self.n, np.uint32)
        k = len(range(t_begin, num_trees, stride))
        stats = np.zeros(4 * max(k, 1), np.uint64)
        rc = lib().or_balance_m(self._h, t_begin, num_trees, stride, seed, sampler, _p(cnt),
                                _p(agree), _p(stats))
        if rc != OR_OK:
            raise OracleError(rc, "or_balance")
        if with_stats:
            return cnt[: self.m], agree, stats[: 4 * k].reshape(k, 4)
        return cnt[: self.m], agree
