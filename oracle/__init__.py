"""CPU oracle for exact triangle counting — TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` leg may import this module.  The
product path (``paper_conf_ipps_li0ptz24_b200``) never imports it, and it
never imports the product path; both take their inputs from ``tcgen``.

The arithmetic lives in ``oracle/tc_oracle.cpp`` (plain C++17 + std::thread,
node-iterator with ``std::set_intersection``; each step cites PAPER.md).
This wrapper only marshals arguments.  Pins: ``tests/test_oracle_pins.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libtcoracle.so")
_lib = None

ORDER_DEGREE, ORDER_ID, ORDER_HASH = 0, 1, 2


class _Result(ctypes.Structure):
    _fields_ = [
        ("triangles", ctypes.c_uint64),
        ("m", ctypes.c_int64),
        ("n_active", ctypes.c_int64),
        ("max_out_degree", ctypes.c_int64),
        ("merge_steps_total", ctypes.c_uint64),
        ("merge_steps_counted", ctypes.c_uint64),
        ("build_ms", ctypes.c_double),
        ("count_ms", ctypes.c_double),
        ("threads", ctypes.c_int32),
        ("sampled", ctypes.c_int32),
    ]


@dataclass
class OracleResult:
    triangles: int
    m: int
    n_active: int
    max_out_degree: int
    merge_steps_total: int
    merge_steps_counted: int
    build_ms: float
    count_ms: float
    threads: int
    sampled: bool


def build_lib() -> str:
    """Compile the oracle with g++ (building the checker is not using it)."""
    src = os.path.join(_HERE, "tc_oracle.cpp")
    if not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["g++", "-O3", "-std=c++17", "-fPIC", "-shared", "-pthread",
                               src, "-o", _LIB_PATH])
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build_lib()
        L = ctypes.CDLL(_LIB_PATH)
        L.tco_count.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                                ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.POINTER(_Result)]
        L.tco_count.restype = ctypes.c_int
        L.tco_build.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                                ctypes.c_int]
        L.tco_build.restype = ctypes.c_void_p
        L.tco_count_rows.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int64,
                                     ctypes.c_int64, ctypes.POINTER(_Result)]
        L.tco_count_rows.restype = ctypes.c_int
        L.tco_free.argtypes = [ctypes.c_void_p]
        L.tco_free.restype = None
        _lib = L
    return _lib


def _wrap(r) -> OracleResult:
    return OracleResult(int(r.triangles), int(r.m), int(r.n_active), int(r.max_out_degree),
                        int(r.merge_steps_total), int(r.merge_steps_counted), float(r.build_ms),
                        float(r.count_ms), int(r.threads), bool(r.sampled))


class OracleGraph:
    """Steps 1-4 done once (tco_build); count_rows() runs step 5 over all rows
    or over the sampled rows x % stride == offset (bench reference leg)."""

    def __init__(self, src, dst, n: int = -1, order: int = ORDER_DEGREE):
        src = np.ascontiguousarray(src, dtype=np.int32)
        dst = np.ascontiguousarray(dst, dtype=np.int32)
        if src.shape != dst.shape:
            raise ValueError("src and dst differ in length")
        self._h = lib().tco_build(src.ctypes.data_as(ctypes.c_void_p),
                                  dst.ctypes.data_as(ctypes.c_void_p), len(src), int(n),
                                  int(order))
        if not self._h:
            raise ValueError("oracle: invalid input (vertex id out of range)")

    def count_rows(self, threads: int = 0, stride: int = 1, offset: int = 0) -> OracleResult:
        r = _Result()
        if lib().tco_count_rows(self._h, int(threads), int(stride), int(offset),
                                ctypes.byref(r)) != 0:
            raise ValueError("oracle: bad arguments")
        return _wrap(r)

    def close(self):
        if self._h:
            lib().tco_free(self._h)
        self._h = None

    def __del__(self):
        self.close()


def count(src, dst, n: int = -1, order: int = ORDER_DEGREE, threads: int = 0,
          sample_stride: int = 1) -> OracleResult:
    """Exact T of the cleaned simple graph given by raw pairs (src[i], dst[i]).

    Raises ValueError on an id outside [0, n).
    """
    src = np.ascontiguousarray(src, dtype=np.int32)
    dst = np.ascontiguousarray(dst, dtype=np.int32)
    if src.shape != dst.shape:
        raise ValueError("src and dst differ in length")
    r = _Result()
    rc = lib().tco_count(src.ctypes.data_as(ctypes.c_void_p), dst.ctypes.data_as(ctypes.c_void_p),
                         len(src), int(n), int(order), int(threads), int(sample_stride),
                         ctypes.byref(r))
    if rc != 0:
        raise ValueError("oracle: invalid input (vertex id out of range)")
    return _wrap(r)


def triangles(src, dst, n: int = -1, **kw) -> int:
    return count(src, dst, n, **kw).triangles


# ---------------------------------------------------------------- per-edge support (f1)

def _support_lib():
    L = lib()
    if not hasattr(L, "_support_ready"):
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        L.tco_support_build.argtypes = [vp, vp, i64, i64]
        L.tco_support_build.restype = vp
        L.tco_support_m.argtypes = [vp]
        L.tco_support_m.restype = i64
        L.tco_support_free.argtypes = [vp]
        L.tco_support_free.restype = None
        L.tco_support_all.argtypes = [vp, ctypes.c_int, vp, vp, vp]
        L.tco_support_all.restype = ctypes.c_int
        L.tco_support_pairs.argtypes = [vp, vp, vp, i64, vp]
        L.tco_support_pairs.restype = ctypes.c_int
        L._support_ready = True
    return L


class SupportGraph:
    """sup(a,b) = |N(a) ∩ N(b)| for the edges {a,b} of the cleaned simple graph
    (tco_support_* in tc_oracle.cpp)."""

    def __init__(self, src, dst, n: int = -1):
        src = np.ascontiguousarray(src, dtype=np.int32)
        dst = np.ascontiguousarray(dst, dtype=np.int32)
        if src.shape != dst.shape:
            raise ValueError("src and dst differ in length")
        self._h = _support_lib().tco_support_build(src.ctypes.data_as(ctypes.c_void_p),
                                                   dst.ctypes.data_as(ctypes.c_void_p),
                                                   len(src), int(n))
        if not self._h:
            raise ValueError("oracle: invalid input (vertex id out of range)")
        self.m = int(_support_lib().tco_support_m(self._h))

    def all(self, threads: int = 0):
        """(a, b, sup): int32, int32, uint32 arrays of length m, ascending (a, b), a < b."""
        a = np.empty(self.m, np.int32)
        b = np.empty(self.m, np.int32)
        s = np.empty(self.m, np.uint32)
        vp = ctypes.c_void_p
        if _support_lib().tco_support_all(self._h, int(threads), a.ctypes.data_as(vp),
                                          b.ctypes.data_as(vp), s.ctypes.data_as(vp)) != 0:
            raise ValueError("oracle: bad arguments")
        return a, b, s

    def pairs(self, a, b):
        """int64 per pair: its support if {a_i, b_i} is an edge, else -1."""
        a = np.ascontiguousarray(a, dtype=np.int32)
        b = np.ascontiguousarray(b, dtype=np.int32)
        out = np.empty(len(a), np.int64)
        vp = ctypes.c_void_p
        if _support_lib().tco_support_pairs(self._h, a.ctypes.data_as(vp), b.ctypes.data_as(vp),
                                            len(a), out.ctypes.data_as(vp)) != 0:
            raise ValueError("oracle: bad arguments")
        return out

    def close(self):
        if self._h:
            _support_lib().tco_support_free(self._h)
        self._h = None

    def __del__(self):
        self.close()


def support(src, dst, n: int = -1, threads: int = 0):
    """Per-edge triangle support of the cleaned simple graph: (a, b, sup) sorted by (a, b)."""
    g = SupportGraph(src, dst, n)
    try:
        return g.all(threads)
    finally:
        g.close()
