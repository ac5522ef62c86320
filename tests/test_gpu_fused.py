"""GPU tests of the library's own cross-GPU sum.

tc_count_range_fused adds each rank's partial count into a symmetric buffer
on every rank — through an NVLS multicast address (multimem.red) or through
the peers' unicast addresses (P2P red over NVLink) — and waits for every
rank.  The GPU box has one B200, so:
  - multicast: a one-device multicast object (tc_mc_buffer_create) exercises
    the multimem.red path on the real NVLS hardware, epoch after epoch;
  - peers: two processes sharing cuda:0, each with the other's buffer mapped
    through CUDA IPC, each counting half of the edges, both must get T.
Every T is compared with the oracle.
"""
import os
import socket

import numpy as np
import pytest

import oracle
import tcgen
from tests import graphs

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


@pytest.mark.parametrize("mode", ["multicast", "peers"])
def test_fused_single_rank_epochs(tc, mode):
    try:
        fs = tc.FusedSum(mode=mode)
    except tc.TCError as e:
        if mode == "multicast" and e.status == tc.TC_ERR_UNSUPPORTED:
            pytest.skip(f"no multicast objects here: {e}")
        raise
    assert fs.mode == mode
    cases = [tcgen.CONFIGS["C1"].generate(1), tcgen.rmat(14, 16, 3)]
    (ks, kd, kn), kt = graphs.complete(3000)  # T = C(3000, 3) > 2^32
    try:
        for src, dst, n in cases:
            want = oracle.triangles(src, dst)
            with tc.build_csr(dev(src), dev(dst), n) as g:
                for _ in range(4):  # epochs alternate the two sum words
                    assert tc.count_partitioned(g, fused=fs) == want
                # partial ranges through the same buffer (world 1: the sum is the range)
                b = g.partition(3)
                parts = [int(fs.count_range(g, b[i], b[i + 1]).item()) for i in range(3)]
                assert sum(parts) == want
        with tc.build_csr(dev(ks), dev(kd), kn) as g:
            assert tc.count_partitioned(g, fused=fs) == kt
        assert fs.epoch == 2 * 7 + 1
    finally:
        fs.close()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, bufs, src, dst, n, epochs, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_li0ptz24_b200 as tc
        fs = tc.FusedSum(peers=bufs)
        out = []
        with tc.build_csr(dev(src), dev(dst), n) as g:
            for _ in range(epochs):
                dist.barrier()
                out.append(tc.count_partitioned(g, fused=fs))
        q.put((rank, out, None))
    except Exception as e:
        q.put((rank, None, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_fused_peers_multi_process(tc, world):
    import torch.multiprocessing as mp
    src, dst, n = tcgen.rmat(15, 16, 5)
    want = oracle.triangles(src, dst)
    bufs = [torch.zeros(tc.FUSED_WORDS, dtype=torch.int64, device="cuda") for _ in range(world)]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, bufs, src, dst, n, 3, q))
             for r in range(world)]
    for p in procs:
        p.start()
    try:
        out = [q.get(timeout=240) for _ in procs]
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    for rank, res, err in out:
        assert err is None, f"rank {rank}: {err}"
        assert res == [want] * 3
    assert int(bufs[0][2].item()) == world * 3  # every rank arrived in every epoch


def test_fused_timeout_poisons(tc, monkeypatch):
    """A peer that never arrives: the last CTA gives up after the arrival bound,
    sets the buffer's POISON word and yields UINT64_MAX; count_partitioned
    raises instead of returning it, and the FusedSum refuses further use."""
    monkeypatch.setenv("TC_FUSED_TIMEOUT_MS", "300")
    src, dst, n = tcgen.CONFIGS["C1"].generate(1)
    own = torch.zeros(tc.FUSED_WORDS, dtype=torch.int64, device="cuda")
    ghost = torch.zeros(tc.FUSED_WORDS, dtype=torch.int64, device="cuda")  # never arrives
    fs = tc.FusedSum(peers=[own, ghost], own=own)
    fs.world = 2
    with tc.build_csr(dev(src), dev(dst), n) as g:
        out = fs.count_range(g, 0, g.m_live)
        assert int(out.item()) & (2**64 - 1) == 2**64 - 1
        assert int(own[3].item()) == 1
        with pytest.raises(tc.TCError):
            fs.check(int(out.item()) & (2**64 - 1))
        assert fs.poisoned
        with pytest.raises(tc.TCError):
            fs.count_range(g, 0, g.m_live)


def test_fused_is_one_launch_fewer(tc):
    """The cross-rank sum runs in the count kernel's last CTA: a fused count of a
    non-empty range launches exactly the count kernels (the ticket word is reset
    for the next launch), an empty range launches the finishing kernel."""
    src, dst, n = tcgen.rmat(14, 16, 3)
    want = oracle.triangles(src, dst)
    fs = tc.FusedSum(mode="peers")
    with tc.build_csr(dev(src), dev(dst), n, options={"long_min": 32}) as g:
        assert g.launches_per_count == 2
        for _ in range(3):
            assert tc.count_partitioned(g, fused=fs) == want
            assert int(fs._keep[0][4].item()) == 0  # grid-completion ticket reset
        assert int(fs.count_range(g, 0, 0).item()) == 0  # empty range: finishing kernel
    fs.close()
