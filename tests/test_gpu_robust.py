"""Boundary and failure-path robustness of the C-ABI (SURVEY.md §4.3 item 2,
§5; the paper records a surveyed kernel returning wrong counts in one mode,
P:289, and runs that failed, Fig. 11):

  - every allocation of a build + count fails in turn through tc_set_allocator:
    the call returns TC_ERR_OUT_OF_MEMORY, and every block the library got is
    handed back (no leak), after which a normal build still counts right;
  - the two-choice table's failure path (cuckoo insert gives up -> the chunk's
    tables are rebuilt with linear probing) is forced with TC_CUCKOO_KICKS=0,
    proven to run (tc_counters) and still gives the oracle's count.
"""
import ctypes

import numpy as np
import pytest

import oracle
import tcgen

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ALLOC = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
FREE = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)


@pytest.fixture(scope="module")
def tc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_li0ptz24_b200 as tc
    tc.lib()
    return tc


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


class FailingAllocator:
    """torch caching-allocator blocks; allocation number `fail_at` (1-based) fails."""

    def __init__(self, fail_at=0):
        self.fail_at, self.n, self.live = fail_at, 0, {}

        def alloc(nbytes, stream, ctx):
            self.n += 1
            if self.n == self.fail_at:
                return None
            p = torch.cuda.caching_allocator_alloc(max(int(nbytes), 1), stream=int(stream or 0))
            self.live[p] = int(nbytes)
            return p

        def free(p, nbytes, stream, ctx):
            self.live.pop(int(p), None)
            torch.cuda.caching_allocator_delete(int(p))

        self._a, self._f = ALLOC(alloc), FREE(free)

    def install(self, tc):
        assert tc.lib().tc_set_allocator(ctypes.cast(self._a, ctypes.c_void_p),
                                         ctypes.cast(self._f, ctypes.c_void_p), None) == 0


def _build_and_count(tc, src, dst, n, host=False):
    if host:
        g = tc.build_csr_host(src, dst, n, options={"long_min": 32})
    else:
        g = tc.build_csr(dev(src), dev(dst), n, options={"long_min": 32})
    try:
        return g.count()
    finally:
        g.close()


@pytest.mark.parametrize("host", [False, True])
def test_every_allocation_failure_is_clean(tc, host):
    src, dst, n = tcgen.rmat(12, 16, 4)
    want = oracle.triangles(src, dst, n)
    probe = FailingAllocator()
    probe.install(tc)
    try:
        assert _build_and_count(tc, src, dst, n, host) == want
        torch.cuda.synchronize()
        total = probe.n
        assert total > 5 and not probe.live
        for k in range(1, total + 1):
            fa = FailingAllocator(k)
            fa.install(tc)
            with pytest.raises(tc.OutOfMemory):
                _build_and_count(tc, src, dst, n, host)
            torch.cuda.synchronize()
            assert not fa.live, f"allocation {k}/{total} failed: {len(fa.live)} blocks leaked"
    finally:
        assert tc.lib().tc_set_allocator(None, None, None) == 0
    assert _build_and_count(tc, src, dst, n, host) == want  # the default allocator again


@pytest.mark.parametrize("graph", ["rmat14", "k_1200"])
def test_cuckoo_failure_rebuilds_linear(tc, monkeypatch, graph):
    if graph == "rmat14":
        src, dst, n = tcgen.rmat(14, 16, 2)
    else:
        from tests import graphs
        (src, dst, n), _ = graphs.complete(1200)
    want = oracle.triangles(src, dst, n)
    opts = {"long_min": 32, "bitmap_factor": -1}  # hash tables only
    tc.counters(reset=True)
    with tc.build_csr(dev(src), dev(dst), n, options=opts) as g:
        assert g.count() == want
    normal = tc.counters(reset=True)["cuckoo_rebuilds"]
    monkeypatch.setenv("TC_CUCKOO_KICKS", "0")  # read when the plan is built
    with tc.build_csr(dev(src), dev(dst), n, options=opts) as g:
        assert g.count() == want
        forced = tc.counters(reset=True)["cuckoo_rebuilds"]
        sup = g.support()
        assert int(sup.to(torch.int64).sum().item()) == 3 * want
        assert tc.counters(reset=True)["cuckoo_rebuilds"] > 0  # the support kernel's path too
    monkeypatch.delenv("TC_CUCKOO_KICKS")
    with tc.build_csr(dev(src), dev(dst), n, options=opts) as g:
        ref = g.support()
        assert torch.equal(ref, sup)
    assert forced > normal and forced > 0
