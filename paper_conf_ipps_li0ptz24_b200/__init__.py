"""b200tc — B200-native intersection-based triangle counting (ITC).

Thin Python binding over the C-ABI in ``include/tc.h`` (``libtc.so``, built
in-tree by ``make`` / ``__graft_entry__.build()``).  This module only
marshals arguments: every step of the path (cleaning, orientation, CSR,
plan, counting, reduction) runs in the library's sm_100a kernels.  PyTorch
supplies device memory for the inputs, the current CUDA stream, and the
process group of :func:`count_partitioned`.

There is no CPU fallback: if ``libtc.so`` is missing or no CUDA device is
present, the entry points raise.

    g = build_csr(src, dst)          # torch int32 CUDA tensors (raw edge list)
    t = g.count()                    # exact uint64 triangle count (int)
    t = count_partitioned(g, group)  # torch.distributed over NCCL
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libtc.so")

TC_OK, TC_ERR_INVALID_ARGUMENT, TC_ERR_OUT_OF_MEMORY, TC_ERR_CUDA, TC_ERR_UNSUPPORTED = range(5)
TC_KEEP_ISOLATED = 0x1

# Every symbol include/tc.h declares (tests check the library exports them).
EXPORTS = (
    "tc_set_allocator", "tc_build_csr", "tc_build_csr_host", "tc_replan", "tc_graph_info",
    "tc_count", "tc_count_async", "tc_count_range", "tc_partition", "tc_partition_prefix",
    "tc_free", "tc_last_error", "tc_version", "tc_support", "tc_edge_list",
    "tc_count_variant", "tc_key_bits", "tc_shard_canon", "tc_shard_histogram", "tc_shard_cuts",
    "tc_shard_bounds", "tc_shard_unique", "tc_shard_degree", "tc_rank_vertices", "tc_shard_orient", "tc_sort_keys",
    "tc_build_from_oriented", "tc_count_range_fused", "tc_mc_buffer_create",
    "tc_mc_buffer_destroy", "tc_partition_measured", "tc_calibrate", "tc_plan_chunks",
    "tc_partition_chunks", "tc_slice_bounds", "tc_counters", "tc_refine_profile",
    "tc_release_memory",
)
TC_MAX_PEERS = 16
CALIBRATION_SLICES = 64  # slices of the measured time profile (tc_calibrate)
FUSED_WORDS = 8  # u64 words of the f4 symmetric buffer (tc_fused.cuh: sums, arrivals, poison, ticket)
VARIANTS = {"polak": 1, "trust": 2}  # tc_count_variant


class TCError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"tc status {status}: {msg}")
        self.status = status


class InvalidArgument(TCError, ValueError):
    pass


class OutOfMemory(TCError, MemoryError):
    pass


class Options(ctypes.Structure):
    """tc_options (0 = library default).  Performance knobs only: they never
    change the count."""
    _fields_ = [("chunk_cost", ctypes.c_int32), ("seg_cost", ctypes.c_int32),
                ("huge_degree", ctypes.c_int32), ("block_threads", ctypes.c_int32),
                ("table_factor", ctypes.c_int32), ("long_min", ctypes.c_int32),
                ("probe_mode", ctypes.c_int32), ("bitmap_factor", ctypes.c_int32)]


class GraphInfo(ctypes.Structure):
    _fields_ = [("n_input", ctypes.c_int64), ("n", ctypes.c_int64), ("m", ctypes.c_int64),
                ("max_out_degree", ctypes.c_int64), ("m_live", ctypes.c_int64),
                ("n_groups", ctypes.c_int64), ("n_chunks", ctypes.c_int64),
                ("keys_total", ctypes.c_int64), ("b_itc", ctypes.c_uint64),
                ("smem_bytes", ctypes.c_int64), ("count_grid", ctypes.c_int32),
                ("count_block", ctypes.c_int32), ("row_ptr", ctypes.c_void_p),
                ("col", ctypes.c_void_p), ("perm", ctypes.c_void_p),
                ("ms_canon", ctypes.c_float), ("ms_sort_unique", ctypes.c_float),
                ("ms_degree_rank", ctypes.c_float), ("ms_orient_csr", ctypes.c_float),
                ("ms_plan", ctypes.c_float), ("ms_total", ctypes.c_float),
                ("n_long_chunks", ctypes.c_int64), ("method_bytes", ctypes.c_uint64),
                ("table_words", ctypes.c_int64), ("group_visits", ctypes.c_int64),
                ("m_live_long", ctypes.c_int64), ("method_bytes_long", ctypes.c_uint64),
                ("keys_long", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_
                if k not in ("row_ptr", "col", "perm")}


_lib = None


def lib():
    """Load libtc.so (raises if it was not built — no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `make` or __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        vp, i64, i32, u32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32
        st = ctypes.c_int
        sig = {
            "tc_set_allocator": ([vp, vp, vp], st),
            "tc_build_csr": ([vp, vp, i64, i64, u32, vp, vp, ctypes.POINTER(vp)], st),
            "tc_build_csr_host": ([vp, vp, i64, i64, u32, vp, vp, ctypes.POINTER(vp)], st),
            "tc_replan": ([vp, vp, vp], st),
            "tc_graph_info": ([vp, ctypes.POINTER(GraphInfo)], st),
            "tc_count": ([vp, vp, ctypes.POINTER(ctypes.c_uint64)], st),
            "tc_count_async": ([vp, vp, vp], st),
            "tc_count_range": ([vp, i64, i64, vp, vp], st),
            "tc_partition": ([vp, i32, vp], st),
            "tc_partition_prefix": ([vp, i64, i32, vp], st),
            "tc_partition_measured": ([vp, i32, i32, vp, vp], st),
            "tc_calibrate": ([vp, vp, i32, vp], st),
            "tc_refine_profile": ([vp, vp, i32, i32, vp], st),
            "tc_plan_chunks": ([vp, vp, vp], st),
            "tc_counters": ([vp, i32], st),
            "tc_release_memory": ([], st),
            "tc_partition_chunks": ([vp, vp, i64, i64, i32, vp, i32, vp], st),
            "tc_slice_bounds": ([vp, i64, i64, i32, vp], st),
            "tc_support": ([vp, vp, vp], st),
            "tc_edge_list": ([vp, vp, vp, vp], st),
            "tc_count_variant": ([vp, i32, vp, vp], st),
            "tc_key_bits": ([i64], i32),
            "tc_shard_canon": ([vp, vp, i64, i64, vp, vp, vp], st),
            "tc_shard_histogram": ([vp, i64, i64, i32, vp, vp], st),
            "tc_shard_cuts": ([vp, i64, i32, vp], st),
            "tc_shard_bounds": ([vp, i64, i64, i32, vp, i32, vp, vp], st),
            "tc_shard_unique": ([vp, i64, i64, vp, vp, vp], st),
            "tc_shard_degree": ([vp, i64, i64, vp, vp], st),
            "tc_rank_vertices": ([vp, i64, u32, vp, vp, vp, vp], st),
            "tc_shard_orient": ([vp, i64, i64, vp, i64, vp, vp], st),
            "tc_sort_keys": ([vp, i64, i64, vp], st),
            "tc_build_from_oriented": ([vp, i64, vp, i64, i64, vp, vp, ctypes.POINTER(vp)], st),
            "tc_count_range_fused": ([vp, i64, i64, vp, vp, vp, i32, ctypes.c_uint64, vp, vp], st),
            "tc_mc_buffer_create": ([ctypes.c_size_t, ctypes.POINTER(vp), ctypes.POINTER(vp),
                                     ctypes.POINTER(vp)], st),
            "tc_mc_buffer_destroy": ([vp], None),
            "tc_free": ([vp], None),
            "tc_last_error": ([], ctypes.c_char_p),
            "tc_version": ([], ctypes.c_char_p),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def _check(status: int):
    if status == TC_OK:
        return
    msg = lib().tc_last_error().decode(errors="replace")
    if status == TC_ERR_INVALID_ARGUMENT:
        raise InvalidArgument(status, msg)
    if status == TC_ERR_OUT_OF_MEMORY:
        raise OutOfMemory(status, msg)
    raise TCError(status, msg)


def version() -> str:
    return lib().tc_version().decode()


def _torch():
    import torch
    return torch


def _stream(stream=None) -> int:
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream)


def _options(opts):
    """tc_options* for the C call (None = defaults)."""
    if opts is None:
        return None
    if not isinstance(opts, Options):
        o = Options()
        for k, v in dict(opts).items():
            setattr(o, k, int(v))
        opts = o
    return ctypes.byref(opts)


class _DevArray:
    """Borrowed device array exposed through __cuda_array_interface__."""

    def __init__(self, ptr: int, n: int, typestr: str, owner):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr,
                                         "data": (ptr or 0, False), "version": 3}
        self._owner = owner


class Graph:
    """An oriented CSR + dispatch plan living on one GPU (owns a tc_graph*)."""

    def __init__(self, handle: int):
        self._h = ctypes.c_void_p(handle)
        self.info = self._info()

    # ------------------------------------------------------------ info
    def _info(self) -> GraphInfo:
        gi = GraphInfo()
        _check(lib().tc_graph_info(self._h, ctypes.byref(gi)))
        return gi

    @property
    def n(self) -> int:
        return int(self.info.n)

    @property
    def m(self) -> int:
        return int(self.info.m)

    @property
    def m_live(self) -> int:
        return int(self.info.m_live)

    @property
    def launches_per_count(self) -> int:
        """Kernels one count launches: one per non-empty work class."""
        gi = self.info
        return int(gi.n_long_chunks > 0) + int(gi.n_chunks - gi.n_long_chunks > 0)

    def csr(self):
        """(row_ptr int64[n+1], col int32[m], perm int32[n]) as borrowed CUDA tensors."""
        torch = _torch()
        gi = self.info
        rp = torch.as_tensor(_DevArray(gi.row_ptr, gi.n + 1, "<i8", self), device="cuda")
        col = torch.as_tensor(_DevArray(gi.col, gi.m, "<i4", self), device="cuda")
        perm = torch.as_tensor(_DevArray(gi.perm, gi.n, "<i4", self), device="cuda")
        return rp, col, perm

    # ------------------------------------------------------------ counting
    def count(self, stream=None) -> int:
        """T (exact; synchronises the stream)."""
        out = ctypes.c_uint64(0)
        _check(lib().tc_count(self._h, ctypes.c_void_p(_stream(stream)), ctypes.byref(out)))
        return int(out.value)

    def count_async(self, out=None, stream=None):
        """Stream-ordered T into a 1-element int64 CUDA tensor (u64 bit pattern)."""
        torch = _torch()
        if out is None:
            out = torch.empty(1, dtype=torch.int64, device="cuda")
        _check(lib().tc_count_async(self._h, ctypes.c_void_p(_stream(stream)),
                                    ctypes.c_void_p(out.data_ptr())))
        return out

    def count_variant(self, variant: str, out=None, stream=None):
        """T by the paper's Polak or TRUST kernel (tc_count_variant), stream-ordered
        into a 1-element int64 CUDA tensor (u64 bit pattern)."""
        torch = _torch()
        if out is None:
            out = torch.empty(1, dtype=torch.int64, device="cuda")
        _check(lib().tc_count_variant(self._h, VARIANTS[variant], ctypes.c_void_p(_stream(stream)),
                                      ctypes.c_void_p(out.data_ptr())))
        return out

    def count_range(self, e_begin: int, e_end: int, out=None, stream=None):
        """Partial count of live oriented edges [e_begin, e_end) (plan order)."""
        torch = _torch()
        if out is None:
            out = torch.empty(1, dtype=torch.int64, device="cuda")
        _check(lib().tc_count_range(self._h, int(e_begin), int(e_end),
                                    ctypes.c_void_p(_stream(stream)),
                                    ctypes.c_void_p(out.data_ptr())))
        return out

    # ------------------------------------------------------------ per-edge support (f1)
    def support(self, out=None, stream=None):
        """Triangles containing each CSR edge: int32 CUDA tensor [m] holding the
        uint32 counts (tc_support; stream-ordered).  Pair with edge_list()."""
        torch = _torch()
        if out is None:
            out = torch.empty(self.m, dtype=torch.int32, device="cuda")
        _check(lib().tc_support(self._h, ctypes.c_void_p(_stream(stream)),
                                ctypes.c_void_p(out.data_ptr())))
        return out

    def edge_list(self, stream=None):
        """(u, v) int32 CUDA tensors [m]: original ids of each CSR edge (tc_edge_list)."""
        torch = _torch()
        u = torch.empty(self.m, dtype=torch.int32, device="cuda")
        v = torch.empty(self.m, dtype=torch.int32, device="cuda")
        _check(lib().tc_edge_list(self._h, ctypes.c_void_p(_stream(stream)),
                                  ctypes.c_void_p(u.data_ptr()), ctypes.c_void_p(v.data_ptr())))
        return u, v

    def partition(self, world_size: int, profile=None) -> list:
        """Cost-balanced chunk-aligned cut of [0, m_live): tc_partition (the
        built-in profile), or tc_partition_measured with ``profile`` = the
        per-slice ms of :meth:`calibrate` (the same on every rank)."""
        b = np.zeros(int(world_size) + 1, dtype=np.int64)
        if profile is None:
            _check(lib().tc_partition(self._h, int(world_size), b.ctypes.data_as(ctypes.c_void_p)))
        else:
            ms = np.ascontiguousarray(profile, dtype=np.float64)
            _check(lib().tc_partition_measured(self._h, int(world_size), int(ms.size),
                                               ms.ctypes.data_as(ctypes.c_void_p),
                                               b.ctypes.data_as(ctypes.c_void_p)))
        return [int(x) for x in b]

    def calibrate(self, n_slices: int = CALIBRATION_SLICES, stream=None) -> np.ndarray:
        """The plan's time profile on this device: ms of each of ``n_slices``
        near-equal-cost slices counted alone (tc_calibrate)."""
        ms = np.zeros(int(n_slices), dtype=np.float64)
        _check(lib().tc_calibrate(self._h, ctypes.c_void_p(_stream(stream)), int(n_slices),
                                  ms.ctypes.data_as(ctypes.c_void_p)))
        return ms

    def refine(self, world_size: int, profile, stream=None) -> np.ndarray:
        """The profile refined for world_size ranks (tc_refine_profile): every
        rank's range of its split timed alone, each slice scaled by measured /
        predicted time.  Returns a new array."""
        ms = np.array(profile, dtype=np.float64, copy=True)
        _check(lib().tc_refine_profile(self._h, ctypes.c_void_p(_stream(stream)), int(world_size),
                                       int(ms.size), ms.ctypes.data_as(ctypes.c_void_p)))
        return ms

    def chunks(self):
        """(first live edge of every chunk, plan cost prefix at it): two int64
        numpy arrays of n_chunks + 1 entries (tc_plan_chunks)."""
        nc = int(self.info.n_chunks)
        seg = np.zeros(nc + 1, dtype=np.int64)
        cost = np.zeros(nc + 1, dtype=np.int64)
        _check(lib().tc_plan_chunks(self._h, seg.ctypes.data_as(ctypes.c_void_p),
                                    cost.ctypes.data_as(ctypes.c_void_p)))
        return seg, cost

    def replan(self, options=None, stream=None):
        _check(lib().tc_replan(self._h, _options(options), ctypes.c_void_p(_stream(stream))))
        self.info = self._info()

    # ------------------------------------------------------------ lifetime
    def close(self):
        if self._h is not None and self._h.value:
            lib().tc_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


def build_csr(src, dst, num_vertices: Optional[int] = None, keep_isolated: bool = False,
              options=None, stream=None) -> Graph:
    """a1..a6 from a raw device edge list (torch int32 CUDA tensors of equal length)."""
    torch = _torch()
    if src.shape != dst.shape or src.dim() != 1:
        raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, "src/dst must be 1-D of equal length")
    if src.dtype != torch.int32 or dst.dtype != torch.int32 or not src.is_cuda or not dst.is_cuda:
        raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, "src/dst must be int32 CUDA tensors")
    src, dst = src.contiguous(), dst.contiguous()
    h = ctypes.c_void_p(0)
    _check(lib().tc_build_csr(ctypes.c_void_p(src.data_ptr()), ctypes.c_void_p(dst.data_ptr()),
                              int(src.numel()), -1 if num_vertices is None else int(num_vertices),
                              TC_KEEP_ISOLATED if keep_isolated else 0, _options(options),
                              ctypes.c_void_p(_stream(stream)), ctypes.byref(h)))
    return Graph(h.value)


def build_csr_host(src: np.ndarray, dst: np.ndarray, num_vertices: Optional[int] = None,
                   keep_isolated: bool = False, options=None, stream=None) -> Graph:
    """Same from host int32 arrays (numpy, or pinned torch CPU tensors): the
    library performs the host->device copy on the stream."""
    def ptr(a):
        if hasattr(a, "data_ptr"):
            return a.data_ptr(), a.numel()
        a = np.ascontiguousarray(a, dtype=np.int32)
        return a.ctypes.data, a.size
    ps, ns = ptr(src)
    pd, nd = ptr(dst)
    if ns != nd:
        raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, "src/dst differ in length")
    h = ctypes.c_void_p(0)
    _check(lib().tc_build_csr_host(ctypes.c_void_p(ps), ctypes.c_void_p(pd), int(ns),
                                   -1 if num_vertices is None else int(num_vertices),
                                   TC_KEEP_ISOLATED if keep_isolated else 0, _options(options),
                                   ctypes.c_void_p(_stream(stream)), ctypes.byref(h)))
    return Graph(h.value)


def partition_prefix(prefix: Sequence[int], world_size: int) -> list:
    """Host-only cost split (tc_partition_prefix): unit bounds cutting the
    exclusive cost prefix into world_size near-equal contiguous parts."""
    p = np.ascontiguousarray(prefix, dtype=np.int64)
    b = np.zeros(int(world_size) + 1, dtype=np.int64)
    _check(lib().tc_partition_prefix(p.ctypes.data_as(ctypes.c_void_p), len(p) - 1,
                                     int(world_size), b.ctypes.data_as(ctypes.c_void_p)))
    return [int(x) for x in b]


def release_memory():
    """Give the library's cached device memory back to the driver (tc_release_memory)."""
    _check(lib().tc_release_memory())


def counters(reset: bool = False) -> dict:
    """Diagnostic counters of the count kernels on the current device (tc_counters)."""
    h = (ctypes.c_uint64 * 4)()
    _check(lib().tc_counters(h, 1 if reset else 0))
    return {"cuckoo_rebuilds": int(h[0])}


def slice_bounds(cost, n_long_chunks: int, n_slices: int) -> list:
    """Host-only slice bounds of a profile (tc_slice_bounds): first chunk of each slice."""
    cs = np.ascontiguousarray(cost, dtype=np.int64)
    f = np.zeros(int(n_slices) + 1, dtype=np.int64)
    _check(lib().tc_slice_bounds(cs.ctypes.data_as(ctypes.c_void_p), cs.size - 1, int(n_long_chunks),
                                 int(n_slices), f.ctypes.data_as(ctypes.c_void_p)))
    return [int(x) for x in f]


def partition_chunks(seg, cost, n_long_chunks: int, profile, world_size: int) -> list:
    """Host-only profile-weighted chunk split (tc_partition_chunks): seg/cost are
    the n_chunks+1 first-edge and cost-prefix arrays of Graph.chunks(), profile
    the per-slice ms of tc_slice_bounds(len(profile))."""
    sg = np.ascontiguousarray(seg, dtype=np.int64)
    cs = np.ascontiguousarray(cost, dtype=np.int64)
    ms = np.ascontiguousarray(profile, dtype=np.float64)
    if sg.shape != cs.shape or sg.size < 1:
        raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, "seg/cost must have n_chunks + 1 entries")
    b = np.zeros(int(world_size) + 1, dtype=np.int64)
    _check(lib().tc_partition_chunks(sg.ctypes.data_as(ctypes.c_void_p),
                                     cs.ctypes.data_as(ctypes.c_void_p), sg.size - 1,
                                     int(n_long_chunks), int(ms.size),
                                     ms.ctypes.data_as(ctypes.c_void_p), int(world_size),
                                     b.ctypes.data_as(ctypes.c_void_p)))
    return [int(x) for x in b]


class FusedSum:
    """the symmetric buffer of the library's own
    cross-GPU sum (tc_count_range_fused) — no NCCL on the counting path.

    mode "multicast": an NVLS multicast address (one multimem.red per rank);
    mode "peers": every rank's unicast address (one P2P red per peer);
    "auto": multicast when available, else peers.  With more than one rank
    the mapping comes from torch symmetric memory (plumbing: allocation and
    handle exchange); a single process gets a one-device multicast object
    from tc_mc_buffer_create, or a plain device buffer in peers mode.
    """

    def __init__(self, group=None, mode: str = "auto", peers=None, own=None):
        import torch
        import torch.distributed as dist
        if mode not in ("auto", "multicast", "peers"):
            raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, f"unknown mode {mode!r}")
        self.group, self.epoch, self._handle, self._keep = group, 0, None, []
        self.poisoned = False
        on = dist.is_available() and dist.is_initialized()
        self.world = dist.get_world_size(group) if on else 1
        self.rank = dist.get_rank(group) if on else 0
        if self.world > TC_MAX_PEERS:
            raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, f"at most {TC_MAX_PEERS} ranks")
        self.mc, self.own, self.peers = 0, 0, None
        if peers is not None:  # caller-provided mapping (tests: IPC-shared buffers)
            self._keep = list(peers)
            self.peers = [int(t.data_ptr()) for t in peers]
            self.own = int(own.data_ptr()) if own is not None else self.peers[self.rank]
            self.mode = "peers"
            return
        if self.world == 1:
            if mode in ("auto", "multicast"):
                h, uc, mc = ctypes.c_void_p(0), ctypes.c_void_p(0), ctypes.c_void_p(0)
                st = lib().tc_mc_buffer_create(8 * FUSED_WORDS, ctypes.byref(h), ctypes.byref(uc),
                                           ctypes.byref(mc))
                if st == TC_OK:
                    self._handle, self.own, self.mc, self.mode = h, uc.value, mc.value, "multicast"
                    return
                if mode == "multicast":
                    _check(st)
            buf = torch.zeros(FUSED_WORDS, dtype=torch.int64, device="cuda")
            self._keep = [buf]
            self.own = int(buf.data_ptr())
            self.peers = [self.own]
            self.mode = "peers"
            return
        import torch.distributed._symmetric_memory as symm
        buf = symm.empty(FUSED_WORDS, dtype=torch.int64,
                         device=torch.device("cuda", torch.cuda.current_device()))
        buf.zero_()
        torch.cuda.synchronize()
        gname = group.group_name if group is not None else dist.group.WORLD.group_name
        h = symm.rendezvous(buf, gname)
        self._keep = [buf, h]
        self.own = int(buf.data_ptr())
        if mode != "peers" and int(getattr(h, "multicast_ptr", 0) or 0):
            self.mc, self.mode = int(h.multicast_ptr), "multicast"
        elif mode == "multicast":
            raise TCError(TC_ERR_UNSUPPORTED, "no multicast address from symmetric memory")
        else:
            self.peers = [int(p) for p in h.buffer_ptrs]
            self.mode = "peers"
        dist.barrier(group=group)

    def count_range(self, graph, e_begin: int, e_end: int, out=None, stream=None):
        """This rank's partial over [e_begin, e_end) summed over all ranks, into
        a 1-element int64 CUDA tensor (u64 bits; UINT64_MAX if a rank never
        arrived — check with :meth:`check`).  Every rank must call it, in the
        same order.  The count kernel's last CTA does the sum (no extra launch
        unless the range is empty)."""
        torch = _torch()
        if self.poisoned:
            raise TCError(TC_ERR_CUDA, "FusedSum poisoned by an earlier arrival timeout: recreate it")
        if out is None:
            out = torch.empty(1, dtype=torch.int64, device="cuda")
        self.epoch += 1
        peers = None
        if self.peers is not None:
            peers = (ctypes.c_void_p * len(self.peers))(*self.peers)
        _check(lib().tc_count_range_fused(graph._h, int(e_begin), int(e_end),
                                          ctypes.c_void_p(self.own),
                                          ctypes.c_void_p(self.mc or None), peers,
                                          int(self.world), int(self.epoch),
                                          ctypes.c_void_p(_stream(stream)),
                                          ctypes.c_void_p(out.data_ptr())))
        return out

    def check(self, value: int) -> int:
        """Raise if the sum of this epoch timed out (a rank never arrived): the
        kernel then wrote UINT64_MAX and set the buffer's POISON word; the
        buffer stays unusable (a late partial may still land in it)."""
        if value & (2**64 - 1) != 2**64 - 1:
            return value
        torch = _torch()
        word = torch.as_tensor(_DevArray(self.own + 8 * 3, 1, "<i8", self), device="cuda")
        if int(word.item()) != 0:
            self.poisoned = True
            raise TCError(TC_ERR_CUDA, "fused sum: a rank did not arrive within 20 s (buffer poisoned)")
        return value

    def close(self):
        if self._handle is not None:
            lib().tc_mc_buffer_destroy(self._handle)
            self._handle = None
        self._keep = []

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def agreed_profile(graph, group=None, stream=None, n_slices: int = CALIBRATION_SLICES):
    """A time profile every rank agrees on: each rank calibrates (tc_calibrate),
    the ranks' profiles are averaged (one all_reduce), refined for this world
    size (tc_refine_profile) and averaged again, so the bounds are identical on
    every rank.  None when not distributed."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return None
    world = dist.get_world_size(group)
    dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"

    def average(ms):
        t = torch.as_tensor(ms, dtype=torch.float64).to(dev)
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
        return (t.cpu().numpy() / world).astype(np.float64)

    ms = average(graph.calibrate(n_slices, stream=stream))
    # one refinement pass for this world size (each rank times every range on
    # its own GPU; the averages keep the bounds identical on every rank)
    return average(graph.refine(world, ms, stream=stream))


def count_partitioned(graph, group=None, stream=None, fused: Optional[FusedSum] = None,
                      profile="auto") -> int:
    """T over a torch.distributed process group.

    Every rank holds the same replicated graph; rank r counts the live
    oriented edges [b_r, b_{r+1}) of the cost-balanced split
    (tc_partition_measured with ``profile``, the same on every rank; the
    default "auto" measures it once per graph with :func:`agreed_profile` when
    there is more than one rank; None = tc_partition's built-in profile) and a single
    all_reduce(SUM) of the 8-byte partials (ProcessGroupNCCL over NVLink on
    the GPU box) gives T on every rank.  Two's-complement int64 addition is
    bit-identical to uint64 addition mod 2^64.  With ``fused`` (a
    :class:`FusedSum`), the sum is the library's own over NVLink peer memory
    (f4) instead of the NCCL all_reduce.
    """
    import torch.distributed as dist
    on = dist.is_available() and dist.is_initialized()
    world = dist.get_world_size(group) if on else 1
    rank = dist.get_rank(group) if on else 0
    if isinstance(profile, str):
        if profile != "auto":
            raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, f"unknown profile {profile!r}")
        profile = getattr(graph, "_agreed_profile", None)
        if profile is None and world > 1:  # collective: every rank measures once per graph
            profile = agreed_profile(graph, group, stream)
            graph._agreed_profile = profile
    bounds = graph.partition(world) if profile is None else graph.partition(world, profile)
    if fused is not None:  # f4: the library's own sum over NVLink peer memory
        total = fused.count_range(graph, bounds[rank], bounds[rank + 1], stream=stream)
        return fused.check(int(total.item()) & (2**64 - 1))
    partial = graph.count_range(bounds[rank], bounds[rank + 1], stream=stream)
    if on:
        dist.all_reduce(partial, op=dist.ReduceOp.SUM, group=group)
    return int(partial.item()) & (2**64 - 1)


from .sharded import build_csr_sharded, shard_cuts  # noqa: E402  (f2)

__all__ = ["FusedSum", "build_csr_sharded", "shard_cuts", "Graph", "Options", "GraphInfo", "build_csr", "build_csr_host", "count_partitioned",
           "partition_prefix", "partition_chunks", "slice_bounds", "counters", "release_memory", "agreed_profile", "version", "lib", "TCError", "InvalidArgument", "OutOfMemory",
           "EXPORTS", "LIB_PATH"]
