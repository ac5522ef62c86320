"""Seeded synthetic edge-list generators (input side only).

This module is the one piece shared by the CUDA path (tests, bench) and the
CPU oracle (tests): it turns (config, seed) into a raw int32 edge list that may
contain self-loops and duplicate / reversed pairs, like the SNAP files the
paper cleans.  It contains none of the counting arithmetic.

The workload recipes are SURVEY.md §8(d) (configs C1..C5); see DESIGN.md
"Input recipe".  The C implementation is ``tcgen.cpp`` (declared in
``include/tcgen.h``), a counter-based integer generator whose output is a pure
function of its arguments.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libtcgen.so")
_lib = None

# Graph500 initiator (0.57, 0.19, 0.19, 0.05) as cumulative 32-bit thresholds.
GRAPH500 = (0.57, 0.19, 0.19)


def _thresholds(a: float, b: float, c: float):
    s = float(1 << 32)
    return int(a * s), int((a + b) * s), int((a + b + c) * s)


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make` (or __graft_entry__.build())")
        L = ctypes.CDLL(_LIB_PATH)
        i64, u64, u32, i32p = ctypes.c_int64, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p
        L.tcgen_rmat.argtypes = [u64, ctypes.c_int, i64, u32, u32, u32, ctypes.c_int, i32p, i32p]
        L.tcgen_rmat.restype = i64
        L.tcgen_chung_lu.argtypes = [u64, i64, i64, ctypes.c_double, ctypes.c_double, i32p, i32p]
        L.tcgen_chung_lu.restype = i64
        L.tcgen_lattice_capacity.argtypes = [i64]
        L.tcgen_lattice_capacity.restype = i64
        L.tcgen_lattice.argtypes = [u64, i64, u32, u32, i32p, i32p]
        L.tcgen_lattice.restype = i64
        L.tcgen_checksum.argtypes = [i32p, i32p, i64]
        L.tcgen_checksum.restype = u64
        L.tcgen_set_threads.argtypes = [ctypes.c_int]
        L.tcgen_set_threads.restype = None
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _empty(n: int):
    # page-aligned host buffers; callers may pin them with torch if they need to
    return np.empty(n, dtype=np.int32)


def rmat(scale: int, edge_factor: int, seed: int, abc=GRAPH500, permute: bool = True):
    """RMAT / Kronecker pairs.  Returns (src, dst, n)."""
    m = edge_factor << scale
    src, dst = _empty(m), _empty(m)
    ta, tab, tabc = _thresholds(*abc)
    r = lib().tcgen_rmat(seed, scale, edge_factor, ta, tab, tabc, int(permute), _ptr(src), _ptr(dst))
    if r != m:
        raise ValueError("tcgen_rmat: bad arguments")
    return src, dst, 1 << scale


def chung_lu(n: int, num_pairs: int, seed: int, gamma: float = 2.5, w_max: float = 15000.0):
    """Chung-Lu power-law pairs shaped like com-LiveJournal (§8(d) C2).  Returns (src, dst, n)."""
    src, dst = _empty(num_pairs), _empty(num_pairs)
    r = lib().tcgen_chung_lu(seed, n, num_pairs, gamma, w_max, _ptr(src), _ptr(dst))
    if r != num_pairs:
        raise ValueError("tcgen_chung_lu: bad arguments")
    return src, dst, n


def lattice(side: int, seed: int, p_keep: float = 0.6, p_diag: float = 0.05):
    """Road-like triangulated lattice (§8(d) C5).  Returns (src, dst, n)."""
    cap = lib().tcgen_lattice_capacity(side)
    src, dst = _empty(cap), _empty(cap)
    s = float(1 << 32)
    r = lib().tcgen_lattice(seed, side, min(int(p_keep * s), 0xFFFFFFFF),
                            min(int(p_diag * s), 0xFFFFFFFF), _ptr(src), _ptr(dst))
    if r < 0:
        raise ValueError("tcgen_lattice: bad arguments")
    return src[:r].copy(), dst[:r].copy(), side * side


def checksum(src: np.ndarray, dst: np.ndarray) -> int:
    src = np.ascontiguousarray(src, dtype=np.int32)
    dst = np.ascontiguousarray(dst, dtype=np.int32)
    return int(lib().tcgen_checksum(_ptr(src), _ptr(dst), len(src)))


@dataclass(frozen=True)
class Config:
    """One BASELINE.json workload."""
    name: str
    kind: str
    params: tuple
    description: str

    def generate(self, seed: int = 1):
        if self.kind == "rmat":
            scale, ef = self.params[:2]
            abc = self.params[2] if len(self.params) > 2 else GRAPH500
            return rmat(scale, ef, seed, abc)
        if self.kind == "chung_lu":
            n, pairs = self.params
            return chung_lu(n, pairs, seed)
        if self.kind == "lattice":
            (side,) = self.params
            return lattice(side, seed)
        raise ValueError(self.kind)


CONFIGS = {
    "C1": Config("C1", "rmat", (10, 16), "RMAT scale-10 ef16 (Graph500 initiator), 16,384 pairs"),
    "C2": Config("C2", "chung_lu", (4_000_000, 35_500_000),
                 "Chung-Lu gamma=2.5 w_max=15000, n=4M, 35.5M pairs (com-LiveJournal-shaped)"),
    "C3": Config("C3", "rmat", (24, 16), "RMAT scale-24 ef16 (Graph500 initiator), 268,435,456 pairs"),
    "C4": Config("C4", "rmat", (26, 24), "Kronecker scale-26 ef24 (Graph500 initiator), ~1.61B pairs"),
    "C5": Config("C5", "lattice", (4899,),
                 "road-like lattice side 4899 (n=24,000,201), p_keep=0.6, p_diag=0.05"),
}
