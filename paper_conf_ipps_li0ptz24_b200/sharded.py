"""Sharded preprocessing.

P ranks, each holding 1/P of the raw pairs, build the SAME replicated graph
that :func:`build_csr` builds from the union of the pairs, while the heavy
sorts run on about 1/P of the keys each:

    local    a1 + a2   tc_shard_canon       sorted unique canonical keys
    exchange           range split by key (histogram -> all_reduce -> cuts ->
                       bounds -> all_to_all): equal keys meet on one rank
    local    a2 + a3   tc_shard_unique      global dedup + partial degrees
                       (one rank: tc_shard_degree only)
    exchange           all_reduce(SUM) of the degrees
    local    a4        tc_rank_vertices     identical on every rank
    local    a5        tc_shard_orient      relabel + orient + sort
    exchange           range split by row of the oriented keys
    local              tc_sort_keys         this rank's rows, sorted
    exchange           all-gather: rank r's rows precede rank r+1's, so the
                       concatenation is the globally sorted key array
    local    a5 + a6   tc_build_from_oriented   CSR + plan

This module only orchestrates: every step on the data runs in libtc.so
(``NativeSteps`` marshals the calls), the exchanges are torch.distributed
collectives (ProcessGroupNCCL over NVLink on the GPU box).  With a gloo group
the collectives are staged through host memory (tests: two ranks sharing one
GPU).  Without an initialised process group it runs as a single rank.
"""
from __future__ import annotations

import ctypes
from typing import Optional

import numpy as np

HIST_BITS = 16  # buckets of the range split (65,536 x 8 B all_reduce)


def shard_cuts(hist, world_size: int) -> list:
    """tc_shard_cuts (host only): bucket cuts with near-equal key counts."""
    from . import _check, lib
    h = np.ascontiguousarray(hist, dtype=np.int64)
    c = np.zeros(int(world_size) + 1, dtype=np.int64)
    _check(lib().tc_shard_cuts(h.ctypes.data_as(ctypes.c_void_p), len(h), int(world_size),
                               c.ctypes.data_as(ctypes.c_void_p)))
    return [int(x) for x in c]


class NativeSteps:
    """The device steps of the sharded build: argument marshalling over the
    tc_shard_* C-ABI (keys are int64 CUDA tensors holding the uint64 bits)."""

    def __init__(self, stream=None):
        import torch
        self.torch = torch
        self.s = ctypes.c_void_p(int((stream or torch.cuda.current_stream()).cuda_stream))

    def _p(self, t):
        return ctypes.c_void_p(t.data_ptr())

    def key_bits(self, n: int) -> int:
        from . import lib
        return int(lib().tc_key_bits(int(n)))

    def canon(self, src, dst, n: int):
        from . import _check, lib
        keys = self.torch.empty(max(src.numel(), 1), dtype=self.torch.int64, device=src.device)
        cnt = ctypes.c_int64(0)
        _check(lib().tc_shard_canon(self._p(src), self._p(dst), int(src.numel()), int(n), self.s,
                                    self._p(keys), ctypes.byref(cnt)))
        return keys[:cnt.value]

    def histogram(self, keys, n: int, hist_bits: int):
        from . import _check, lib
        hist = self.torch.empty(1 << hist_bits, dtype=self.torch.int64, device=keys.device)
        _check(lib().tc_shard_histogram(self._p(keys), int(keys.numel()), int(n), int(hist_bits),
                                        self.s, self._p(hist)))
        return hist

    def cuts(self, hist_host: np.ndarray, world: int) -> list:
        return shard_cuts(hist_host, world)

    def bounds(self, keys, n: int, hist_bits: int, cuts: list) -> list:
        from . import _check, lib
        c = np.ascontiguousarray(cuts, dtype=np.int64)
        b = np.zeros(len(cuts), dtype=np.int64)
        _check(lib().tc_shard_bounds(self._p(keys), int(keys.numel()), int(n), int(hist_bits),
                                     c.ctypes.data_as(ctypes.c_void_p), len(cuts) - 1, self.s,
                                     b.ctypes.data_as(ctypes.c_void_p)))
        return [int(x) for x in b]

    def degree_buffer(self, n: int, device):
        return self.torch.zeros(max(n, 1), dtype=self.torch.int32, device=device)

    def unique(self, keys, n: int, deg):
        from . import _check, lib
        cnt = ctypes.c_int64(0)
        _check(lib().tc_shard_unique(self._p(keys), int(keys.numel()), int(n), self.s,
                                     ctypes.byref(cnt), self._p(deg)))
        return keys[:cnt.value]

    def degree(self, keys, n: int, deg):
        from . import _check, lib
        _check(lib().tc_shard_degree(self._p(keys), int(keys.numel()), int(n), self.s,
                                     self._p(deg)))

    def rank(self, deg, n: int, flags: int):
        from . import _check, lib
        rank = self.torch.empty(max(n, 1), dtype=self.torch.int32, device=deg.device)
        perm = self.torch.empty(max(n, 1), dtype=self.torch.int32, device=deg.device)
        na = ctypes.c_int64(0)
        _check(lib().tc_rank_vertices(self._p(deg), int(n), int(flags), self.s, self._p(rank),
                                      self._p(perm), ctypes.byref(na)))
        return rank, perm, int(na.value)

    def orient(self, keys, n: int, rank, n_act: int):
        from . import _check, lib
        okeys = self.torch.empty(max(keys.numel(), 1), dtype=self.torch.int64, device=keys.device)
        _check(lib().tc_shard_orient(self._p(keys), int(keys.numel()), int(n), self._p(rank),
                                     int(n_act), self.s, self._p(okeys)))
        return okeys[:keys.numel()]

    def sort(self, keys, n: int):
        from . import _check, lib
        _check(lib().tc_sort_keys(self._p(keys), int(keys.numel()), int(n), self.s))
        return keys

    def build(self, okeys, perm, n_act: int, n_input: int, options=None):
        from . import Graph, _check, _options, lib
        h = ctypes.c_void_p(0)
        _check(lib().tc_build_from_oriented(self._p(okeys), int(okeys.numel()), self._p(perm),
                                            int(n_act), int(n_input), _options(options), self.s,
                                            ctypes.byref(h)))
        return Graph(h.value)


class _Comm:
    """The collectives of the sharded build over one process group (or none:
    a single rank).  Device tensors go straight to NCCL; a gloo group gets
    host copies (gloo's all_to_all is CPU-only)."""

    def __init__(self, group=None):
        import torch
        import torch.distributed as dist
        self.torch, self.dist, self.group = torch, dist, group
        self.on = dist.is_available() and dist.is_initialized()
        self.world = dist.get_world_size(group) if self.on else 1
        self.rank = dist.get_rank(group) if self.on else 0
        self.host = self.on and dist.get_backend(group) == "gloo"

    def _to(self, t):
        return t.cpu() if self.host else t

    def all_reduce(self, t):
        if self.world == 1:
            return t
        x = self._to(t)
        self.dist.all_reduce(x, op=self.dist.ReduceOp.SUM, group=self.group)
        if x is not t:
            t.copy_(x)
        return t

    def all_to_all_v(self, t, send: list):
        """Rank r receives send_q[r] elements from every rank q, in rank order."""
        if self.world == 1:
            return t
        torch = self.torch
        sc = self._to(torch.tensor(send, dtype=torch.int64, device=t.device))
        rc = torch.empty_like(sc)
        self.dist.all_to_all_single(rc, sc, group=self.group)
        recv = [int(x) for x in rc.tolist()]
        x = self._to(t)
        out = torch.empty(sum(recv), dtype=t.dtype, device=x.device)
        self.dist.all_to_all_single(out, x, output_split_sizes=recv, input_split_sizes=send,
                                    group=self.group)
        return out.to(t.device) if self.host else out

    def all_gather_v(self, t):
        """Concatenation of every rank's t, in rank order (one broadcast per
        rank into its slot of the output: NCCL all_gather needs equal sizes)."""
        if self.world == 1:
            return t
        torch = self.torch
        cnt = self._to(torch.tensor([t.numel()], dtype=torch.int64, device=t.device))
        cnts = [torch.empty_like(cnt) for _ in range(self.world)]
        self.dist.all_gather(cnts, cnt, group=self.group)
        sizes = [int(c.item()) for c in cnts]
        x = self._to(t)
        out = torch.empty(sum(sizes), dtype=t.dtype, device=x.device)
        off = 0
        for r, k in enumerate(sizes):
            view = out[off:off + k]
            if r == self.rank:
                view.copy_(x)
            src = self.dist.get_global_rank(self.group, r) if self.group is not None else r
            self.dist.broadcast(view, src=src, group=self.group)
            off += k
        return out.to(t.device) if self.host else out


def _range_exchange(keys, nbound: int, steps, comm: _Comm):
    """Redistribute sorted keys so rank r holds the r-th contiguous key range
    (near-equal sizes by a global histogram of the top key bits)."""
    if comm.world == 1:
        return keys
    hb = min(HIST_BITS, 2 * steps.key_bits(nbound))
    hist = comm.all_reduce(steps.histogram(keys, nbound, hb))
    cuts = steps.cuts(hist.cpu().numpy(), comm.world)
    b = steps.bounds(keys, nbound, hb, cuts)
    return comm.all_to_all_v(keys, [b[r + 1] - b[r] for r in range(comm.world)])


def build_csr_sharded(src, dst, num_vertices: int, group=None, keep_isolated: bool = False,
                      options=None, stream=None, steps=None, timings: Optional[dict] = None):
    """The replicated graph of the union of every rank's (src, dst) shard.

    src, dst: this rank's raw pairs (int32 CUDA tensors, equal length, any
    split of the edge list across ranks).  num_vertices: the common vertex
    bound (required: all ranks must key the same way).  Returns a
    :class:`Graph` equal, byte for byte in its CSR, to ``build_csr`` of the
    concatenated pairs.  ``timings`` (optional dict) receives host wall ms
    per phase (after a stream sync at each phase end).  ``stream``: the
    CUDA stream of every step; it is made torch's current stream for the
    duration, so the collectives are ordered after the native steps.
    """
    import time
    import torch
    from . import TC_KEEP_ISOLATED, InvalidArgument, TC_ERR_INVALID_ARGUMENT
    if num_vertices is None or int(num_vertices) < 0:
        raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, "build_csr_sharded needs num_vertices >= 0")
    if src.shape != dst.shape or src.dim() != 1:
        raise InvalidArgument(TC_ERR_INVALID_ARGUMENT, "src/dst must be 1-D of equal length")
    if stream is not None and steps is None:
        # the collectives order after torch's CURRENT stream: make the given
        # stream current for the whole build so the native steps (enqueued on
        # it) and the collectives are ordered with each other
        with torch.cuda.stream(stream):
            return build_csr_sharded(src, dst, num_vertices, group, keep_isolated, options,
                                     None, None, timings)
    n = int(num_vertices)
    steps = steps or NativeSteps(stream)
    comm = _Comm(group)
    t0 = [time.perf_counter()]

    def mark(name):
        if timings is not None:
            if torch.cuda.is_available() and src.is_cuda:
                torch.cuda.current_stream().synchronize()
            t = time.perf_counter()
            timings[name] = (t - t0[0]) * 1e3
            t0[0] = t

    keys = steps.canon(src.contiguous(), dst.contiguous(), n)
    mark("canon_sort")
    keys = _range_exchange(keys, n, steps, comm)
    mark("exchange1")
    deg = steps.degree_buffer(n, keys.device)
    if comm.world > 1:
        keys = steps.unique(keys, n, deg)
        comm.all_reduce(deg)
    else:  # one rank: tc_shard_canon's keys are already globally sorted and unique
        steps.degree(keys, n, deg)
    mark("unique_degree")
    rank, perm, n_act = steps.rank(deg, n, TC_KEEP_ISOLATED if keep_isolated else 0)
    del deg
    okeys = steps.orient(keys, n, rank, n_act)
    del keys, rank
    mark("rank_orient")
    okeys = _range_exchange(okeys, n_act, steps, comm)
    if comm.world > 1:
        okeys = steps.sort(okeys, n_act)
    mark("exchange2_sort")
    full = comm.all_gather_v(okeys)
    del okeys
    mark("all_gather")
    g = steps.build(full, perm[:n_act], n_act, n, options)
    mark("csr_plan")
    return g
