"""CPU-side checks of the C-ABI library: it loads, exports every symbol that
include/graphb.h declares, its host-only hash self test passes, and argument
/ state errors are reported without touching a GPU."""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_sc_alabanditrb21_b200 import _build, graphb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    _build.build()


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "graphb.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gb_[a-z_]+)\s*\(", src)))


def test_header_symbols_exported():
    L = ctypes.CDLL(_build.LIB)
    syms = declared_symbols()
    assert "gb_load_csr" in syms and "gb_balance" in syms and "gb_free" in syms
    for s in syms:
        assert hasattr(L, s), s
    assert sorted(graphb.exported_symbols()) == syms


def test_sm100a_cubin_in_library():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", _build.LIB], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_selftest_hash_and_decode():
    assert graphb.lib().gb_selftest() == 0


def test_state_and_argument_errors_without_gpu():
    L = graphb.lib()
    graphb.free()
    cnt = np.zeros(4, np.uint32)
    assert L.gb_balance(1, 1, cnt.ctypes.data, cnt.ctypes.data) == graphb.GB_ESTATE
    rp = np.array([0, 1, 2], np.int64)
    col = np.array([1, 0], np.int32)
    sg = np.array([1, 1], np.int8)
    # invalid sizes are rejected before any device work
    assert L.gb_load_csr(0, 1, rp.ctypes.data, col.ctypes.data, sg.ctypes.data) == graphb.GB_EINVAL
    assert L.gb_load_csr(2, 2, rp.ctypes.data, col.ctypes.data, sg.ctypes.data) == graphb.GB_EINVAL
    assert L.gb_load_csr(2, 1, rp.ctypes.data, None, None) == graphb.GB_EINVAL
    assert L.gb_set_option(b"nope", 1) == graphb.GB_EINVAL
    assert L.gb_set_option(b"walk", 4) == graphb.GB_EINVAL          # two-ended, Alg. 3, paper lists, pre climb
    assert L.gb_set_option(b"graphs", 1) == graphb.GB_EINVAL        # not an option (never implemented)
    assert L.gb_set_option(b"sampler", 3) == graphb.GB_EINVAL      # BFS, uniform, DFS only
    assert L.gb_set_option(b"sampler", -1) == graphb.GB_EINVAL
    assert L.gb_set_option(b"jump", 3) == graphb.GB_EINVAL         # 1, 2 or 4 levels
    for k, v in [(b"sampler", 2), (b"wilson", 1), (b"harary", 1), (b"jump", 4), (b"recpass", 0),
                 (b"walk", 2), (b"walk", 3), (b"desc_linear", 1), (b"walk_ept", 4), (b"push_parent", 0),
                 (b"batch", 128)]:
        assert L.gb_set_option(k, v) == 0
    assert L.gb_set_option(b"reset", 0) == 0
    # label / BFS profiles need the msprof option (and a run)
    buf = np.zeros(1024, np.uint64)
    assert L.gb_label_profile(buf.ctypes.data) == graphb.GB_ESTATE
    assert L.gb_msbfs_profile(buf.ctypes.data) == graphb.GB_ESTATE


@pytest.mark.skipif(__import__("tests.conftest", fromlist=["x"]).cuda_available(),
                    reason="checks the no-GPU error path")
def test_no_cpu_fallback():
    """Without a CUDA device the library refuses (GB_ECUDA); it never computes
    on the host."""
    L = graphb.lib()
    rp = np.array([0, 1, 2], np.int64)
    col = np.array([1, 0], np.int32)
    sg = np.array([1, 1], np.int8)
    assert L.gb_load_csr(2, 1, rp.ctypes.data, col.ctypes.data, sg.ctypes.data) == graphb.GB_ECUDA
    with pytest.raises(graphb.GraphBError):
        graphb.load_csr(rp, col, sg)
