"""world_size-2 gloo test of the count_partitioned glue (-m "not gpu").

The product's count_partitioned runs over ProcessGroupNCCL on the GPU box.
Here a test double stands in for the GPU graph (it sums a fixed per-edge
array over the requested range) so that the partition -> per-rank range ->
all_reduce(SUM) -> uint64 logic is exercised with two real processes on CPU.
SURVEY.md §4.3 item 5 allows gloo only as such a double.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


class FakeGraph:
    """Per-edge counts c_e in chunks of 7 edges (the first 60% "long");
    partition/calibrate/count_range mimic the C-ABI contract.  calibrate()
    returns a rank-dependent profile, so only an agreed (averaged) profile
    gives every rank the same bounds."""

    def __init__(self, per_edge):
        self.c = np.asarray(per_edge, dtype=np.uint64)
        self.m_live = len(self.c)
        self.seg = np.concatenate([np.arange(0, self.m_live, 7), [self.m_live]]).astype(np.int64)
        self.cost = self.seg * 3  # cost units: 3 per edge
        self.n_long = (len(self.seg) - 1) * 6 // 10

    def calibrate(self, n_slices=64, stream=None):
        import torch.distributed as dist
        rng = np.random.default_rng(dist.get_rank() if dist.is_initialized() else 0)
        return rng.uniform(0.5, 2.0, size=n_slices)

    def refine(self, world, profile, stream=None):
        import torch.distributed as dist
        rng = np.random.default_rng(100 + (dist.get_rank() if dist.is_initialized() else 0))
        return np.asarray(profile) * rng.uniform(0.9, 1.1, size=len(profile))

    def partition(self, world, profile=None):
        import paper_conf_ipps_li0ptz24_b200 as tc
        if profile is None:
            prefix = np.concatenate([[0], np.cumsum(self.c.astype(np.int64) + 1)])
            return tc.partition_prefix(prefix, world)
        return tc.partition_chunks(self.seg, self.cost, self.n_long, profile, world)

    def count_range(self, b, e, stream=None):
        s = int(self.c[b:e].sum(dtype=np.uint64))
        return torch.tensor([s - (1 << 64) if s >= 1 << 63 else s], dtype=torch.int64)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, per_edge, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_li0ptz24_b200 as tc
        g = FakeGraph(per_edge)
        t = tc.count_partitioned(g)  # "auto": one agreed (all_reduce-averaged) profile
        q.put((rank, t, g.partition(world, g._agreed_profile)))
    finally:
        dist.destroy_process_group()


def _run(per_edge, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, per_edge, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out)


def test_count_partitioned_two_ranks():
    rng = np.random.default_rng(3)
    per_edge = rng.integers(0, 1000, size=10_000)
    out = _run(per_edge)
    total = int(per_edge.sum())
    assert [r[1] for r in out] == [total, total]
    b = out[0][2]
    assert b[0] == 0 and b[-1] == len(per_edge) and b == out[1][2]  # same bounds on both ranks
    assert set(b) <= set(FakeGraph(per_edge).seg.tolist())  # chunk-aligned


def test_count_partitioned_exceeds_63_bits():
    """The int64 all_reduce must reproduce uint64 sums mod 2^64 (C-13)."""
    per_edge = np.array([2**62, 2**62, 2**62, 5], dtype=np.uint64)
    out = _run(per_edge)
    assert [r[1] for r in out] == [3 * 2**62 + 5] * 2
