"""GPU parity of the sharded build through the C-ABI.

The sharded build must give the SAME graph as tc_build_csr on the union of
the shards: row_ptr, col and perm byte for byte (a4's ranking is a function
of the global degrees only), hence the same count, which is also compared
with the oracle.  Multi-rank runs use two or three processes sharing cuda:0
over gloo (collectives staged through host memory; the GPU box has one GPU),
with uneven and empty shards.
"""
import os
import socket

import numpy as np
import pytest

import oracle
import tcgen

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_li0ptz24_b200 as tc
    tc.lib()
    return tc


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def csr_host(g):
    rp, col, perm = g.csr()
    return rp.cpu().numpy().copy(), col.cpu().numpy().copy(), perm.cpu().numpy().copy()


def split_of(m, world, rank, how):
    idx = np.arange(m)
    if how == "blocks":
        return (idx * world) // max(m, 1) == rank
    if how == "interleaved":
        return (idx * 7 + 3) % (world + 1) % world == rank
    if how == "one_empty":  # rank 0 holds nothing
        return (idx % max(world - 1, 1)) + 1 == rank if world > 1 else idx >= 0
    raise ValueError(how)


@pytest.mark.parametrize("case", ["C1", "rmat14", "C5small", "karate_dups"])
def test_single_rank_sharded_equals_build_csr(tc, golden, case):
    if case == "C1":
        src, dst, n = tcgen.CONFIGS["C1"].generate(1)
    elif case == "rmat14":
        src, dst, n = tcgen.rmat(14, 16, 7)
    elif case == "C5small":
        src, dst, n = tcgen.lattice(300, 3)
    else:
        s, d = golden("karate.txt")
        src = np.concatenate([s, d, s, np.arange(34)]).astype(np.int32)  # dups, reversed, loops
        dst = np.concatenate([d, s, d, np.arange(34)]).astype(np.int32)
        n = 40  # isolated vertices 34..39
    with tc.build_csr(dev(src), dev(dst), n) as g0, \
            tc.build_csr_sharded(dev(src), dev(dst), n) as g1:
        for a, b in zip(csr_host(g0), csr_host(g1)):
            assert np.array_equal(a, b)
        t = g1.count()
        assert t == g0.count() == oracle.triangles(src, dst)
        assert g1.info.b_itc == g0.info.b_itc and g1.m_live == g0.m_live


def test_single_rank_sharded_keep_isolated_and_empty(tc):
    src, dst, n = tcgen.CONFIGS["C1"].generate(2)
    with tc.build_csr(dev(src), dev(dst), n + 5, keep_isolated=True) as g0, \
            tc.build_csr_sharded(dev(src), dev(dst), n + 5, keep_isolated=True) as g1:
        for a, b in zip(csr_host(g0), csr_host(g1)):
            assert np.array_equal(a, b)
        assert g1.n == n + 5
    e = np.zeros(0, dtype=np.int32)
    with tc.build_csr_sharded(dev(e), dev(e), 10) as g:
        assert g.count() == 0 and g.m == 0
    with pytest.raises(tc.InvalidArgument):
        tc.build_csr_sharded(dev([0, 11]), dev([1, 2]), 10)
    with pytest.raises(tc.InvalidArgument):
        tc.build_csr_sharded(dev([0]), dev([1]), None)


# ------------------------------------------------------------------ multi-rank (gloo, shared GPU)

def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, src, dst, n, how, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_li0ptz24_b200 as tc
        mine = split_of(len(src), world, rank, how)
        with tc.build_csr_sharded(dev(src[mine]), dev(dst[mine]), n) as g:
            rp, col, perm = csr_host(g)
            t_part = tc.count_partitioned(g)
            q.put((rank, rp, col, perm, g.count(), t_part))
    except Exception as e:  # surface the failure in the parent
        q.put((rank, repr(e), None, None, None, None))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,how,case", [(2, "blocks", "rmat16"), (3, "interleaved", "rmat16"),
                                            (3, "one_empty", "C1"), (2, "interleaved", "C5small")])
def test_multi_rank_sharded_equals_build_csr(tc, world, how, case):
    import torch.multiprocessing as mp
    if case == "rmat16":
        src, dst, n = tcgen.rmat(16, 16, 11)
    elif case == "C1":
        src, dst, n = tcgen.CONFIGS["C1"].generate(3)
    else:
        src, dst, n = tcgen.lattice(400, 5)
    want_t = oracle.triangles(src, dst)
    with tc.build_csr(dev(src), dev(dst), n) as g0:
        want = csr_host(g0)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, src, dst, n, how, q))
             for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, rp, col, perm, t, t_part in out:
        assert col is not None, f"rank {rank}: {rp}"
        assert np.array_equal(rp, want[0]) and np.array_equal(col, want[1])
        assert np.array_equal(perm, want[2])
        assert t == t_part == want_t
