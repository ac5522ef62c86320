"""world_size 2/3 gloo tests of the sharded-build orchestration (f2, -m "not gpu").

build_csr_sharded's device steps run in libtc.so on the GPU box; here a NumPy
test double (``NumpySteps``) stands in for them so that the exchange logic —
histogram all_reduce, tc_shard_cuts (the real host function), range bounds,
all_to_all_v, degree all_reduce, the second range split and the ordered
all-gather — runs with real processes over gloo on CPU.  The result must equal
the single-rank pipeline on the union of the shards, for any split of the
pairs across ranks (the GPU test compares the real library's CSR byte for
byte with tc_build_csr).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


class NumpySteps:
    """Test double of sharded.NativeSteps on CPU tensors."""

    def key_bits(self, n):
        import paper_conf_ipps_li0ptz24_b200 as tc
        return int(tc.lib().tc_key_bits(int(n)))

    def canon(self, src, dst, n):
        a, b = src.numpy().astype(np.int64), dst.numpy().astype(np.int64)
        assert ((a >= 0) & (a < n) & (b >= 0) & (b < n)).all()
        keep = a != b
        lo, hi = np.minimum(a, b)[keep], np.maximum(a, b)[keep]
        return torch.from_numpy(np.unique((lo << self.key_bits(n)) | hi))

    def histogram(self, keys, n, hb):
        shift = 2 * self.key_bits(n) - hb
        return torch.from_numpy(np.bincount(keys.numpy() >> shift, minlength=1 << hb).astype(np.int64))

    def cuts(self, hist, world):
        import paper_conf_ipps_li0ptz24_b200 as tc
        return tc.shard_cuts(hist, world)

    def bounds(self, keys, n, hb, cuts):
        shift = 2 * self.key_bits(n) - hb
        k = keys.numpy()
        return [0] + [int(np.searchsorted(k, c << shift)) if c < (1 << hb) else len(k)
                      for c in cuts[1:-1]] + [len(k)]

    def degree_buffer(self, n, device):
        return torch.zeros(max(n, 1), dtype=torch.int32)

    def unique(self, keys, n, deg):
        u = np.unique(keys.numpy())
        bits = self.key_bits(n)
        d = deg.numpy()
        np.add.at(d, u >> bits, 1)
        np.add.at(d, u & ((1 << bits) - 1), 1)
        return torch.from_numpy(u)

    def degree(self, keys, n, deg):
        self.unique(keys, n, deg)

    def rank(self, deg, n, flags):
        d = deg.numpy()[:n].astype(np.int64)
        ids = np.arange(n)
        order = np.lexsort((ids, d))
        order = order[d[order] > 0] if not flags else order
        rank = np.full(max(n, 1), -1, dtype=np.int32)
        rank[order] = np.arange(len(order), dtype=np.int32)
        perm = np.zeros(max(n, 1), dtype=np.int32)
        perm[:len(order)] = order
        return torch.from_numpy(rank), torch.from_numpy(perm), len(order)

    def orient(self, keys, n, rank, n_act):
        bits, bits2 = self.key_bits(n), self.key_bits(n_act)
        k = keys.numpy()
        ra = rank.numpy()[k >> bits].astype(np.int64)
        rb = rank.numpy()[k & ((1 << bits) - 1)].astype(np.int64)
        return torch.from_numpy(np.sort((np.minimum(ra, rb) << bits2) | np.maximum(ra, rb)))

    def sort(self, keys, n):
        return torch.from_numpy(np.sort(keys.numpy()))

    def build(self, okeys, perm, n_act, n_input, options=None):
        return okeys.numpy().copy(), perm.numpy().copy(), n_act


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, src, dst, n, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_li0ptz24_b200.sharded import build_csr_sharded
        # uneven, interleaved split of the pairs across the ranks
        idx = np.arange(len(src))
        mine = (idx * 7 + 3) % (world + 1) % world == rank
        s = torch.from_numpy(src[mine].astype(np.int32))
        d = torch.from_numpy(dst[mine].astype(np.int32))
        okeys, perm, n_act = build_csr_sharded(s, d, n, steps=NumpySteps())
        q.put((rank, okeys, perm[:n_act]))
    finally:
        dist.destroy_process_group()


def _run(src, dst, n, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, src, dst, n, q))
             for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=180) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out, key=lambda x: x[0])


def _single(src, dst, n):
    from paper_conf_ipps_li0ptz24_b200.sharded import build_csr_sharded
    okeys, perm, n_act = build_csr_sharded(torch.from_numpy(src.astype(np.int32)),
                                           torch.from_numpy(dst.astype(np.int32)), n,
                                           steps=NumpySteps())
    return okeys, perm[:n_act]


def _graph(seed, n=3000, m=40000):
    rng = np.random.default_rng(seed)
    # skewed ids (hubs), duplicates, reversed pairs and self-loops
    src = (n * rng.random(m) ** 3).astype(np.int64)
    dst = rng.integers(0, n, m)
    dst[:200] = src[:200]
    src = np.concatenate([src, dst[:500]])
    dst = np.concatenate([dst, src[:500]])
    return src, dst, n


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_build_equals_single_rank(world):
    src, dst, n = _graph(world)
    want_keys, want_perm = _single(src, dst, n)
    out = _run(src, dst, n, world)
    for _, okeys, perm in out:
        assert np.array_equal(okeys, want_keys)
        assert np.array_equal(perm, want_perm)
    # the single-rank pipeline is the plain definition: unique undirected edges
    m = len({(min(a, b), max(a, b)) for a, b in zip(src.tolist(), dst.tolist()) if a != b})
    assert len(want_keys) == m


def test_shard_cuts_balance():
    """tc_shard_cuts: contiguous bucket ranges, near-equal counts (host only)."""
    import paper_conf_ipps_li0ptz24_b200 as tc
    rng = np.random.default_rng(0)
    hist = rng.integers(0, 1000, 65536)
    hist[123] = 10**6  # one heavy bucket
    for P in (1, 2, 3, 8):
        c = tc.shard_cuts(hist, P)
        assert c[0] == 0 and c[-1] == len(hist) and all(a <= b for a, b in zip(c, c[1:]))
        parts = [int(hist[c[r]:c[r + 1]].sum()) for r in range(P)]
        assert sum(parts) == int(hist.sum())
        assert max(parts) <= hist.sum() / P + hist.max()
    assert tc.shard_cuts(np.zeros(4, dtype=np.int64), 2)[-1] == 4
    with pytest.raises(tc.InvalidArgument):
        tc.shard_cuts(np.array([1, -1]), 2)
