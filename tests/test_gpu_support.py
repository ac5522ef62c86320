"""GPU parity of the per-edge support: tc_support through
the C-ABI vs the oracle's |N(a) ∩ N(b)| (oracle.support / SupportGraph.pairs),
bit-exact, on the same seeded inputs.  The support of an edge is unique, so the
comparison is edge by edge after mapping CSR positions to original ids with
tc_edge_list and sorting by the canonical pair (a < b).
"""
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


def gpu_support(g):
    """(a, b, sup) of the GPU graph, canonical (a < b) and sorted by (a, b)."""
    sup = g.support().cpu().numpy().view(np.uint32)
    u, v = (x.cpu().numpy() for x in g.edge_list())
    a, b = np.minimum(u, v), np.maximum(u, v)
    order = np.argsort((a.astype(np.int64) << 32) | b, kind="stable")
    return a[order], b[order], sup[order]


def check_full(tc, src, dst, n, **kw):
    want = oracle.support(src, dst, n)
    with tc.build_csr(dev(src), dev(dst), n, **kw) as g:
        got = gpu_support(g)
        t = g.count()
    for x, y in zip(got, want):
        assert np.array_equal(x, y)
    assert int(got[2].sum(dtype=np.int64)) == 3 * t
    return got


@pytest.mark.parametrize("name", ["K3", "K10", "K33", "W10", "F300", "K3,4,5", "K5,6,7,8",
                                  "Q4", "star1000", "petersen"])
@pytest.mark.parametrize("long_min", [None, 32])  # None: small graphs are all short class
def test_closed_forms(tc, name, long_min):
    (src, dst, n), _ = graphs.closed_form_cases()[name]
    check_full(tc, src, dst, n, options=None if long_min is None else {"long_min": long_min})


def test_complete_graph_value(tc):
    (src, dst, n), _ = graphs.complete(60)
    a, b, s = check_full(tc, src, dst, n)
    assert (s == 58).all()


@pytest.mark.parametrize("name,n", [("karate.txt", 34), ("lesmis.txt", 77), ("davis.txt", 32)])
def test_golden(tc, golden, name, n):
    src, dst = golden(name)
    check_full(tc, src, dst, n)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_c1_seeds(tc, seed):
    src, dst, n = tcgen.CONFIGS["C1"].generate(seed)
    check_full(tc, src, dst, n)
    check_full(tc, src, dst, n, options={"long_min": 32})  # with the long (tile) class


@pytest.mark.parametrize("scale,ef,seed", [(14, 16, 1), (16, 16, 2)])
def test_rmat_medium(tc, scale, ef, seed):
    src, dst, n = tcgen.rmat(scale, ef, seed)
    check_full(tc, src, dst, n)


def test_skewed_rmat(tc):
    src, dst, n = tcgen.rmat(15, 16, 4, abc=(0.65, 0.15, 0.15))
    check_full(tc, src, dst, n)


@pytest.mark.parametrize("opts", [
    {"probe_mode": 1},                    # linear-probing tables
    {"bitmap_factor": -1},                # hash tables only
    {"bitmap_factor": 64},                # bitmaps almost everywhere
    {"huge_degree": 16},                  # global binary search for d+(v) > 16
    {"long_min": 1},                      # all edges in the tile class
    {"long_min": 32},                     # the split the large graphs use
    {"long_min": 32, "probe_mode": 1},
    {"long_min": 32, "bitmap_factor": -1},
    {"long_min": 1 << 30},                # all edges flattened
    {"table_factor": 2, "chunk_cost": 256},
])
def test_plan_options_never_change_support(tc, opts):
    src, dst, n = tcgen.rmat(13, 16, 7)
    check_full(tc, src, dst, n, options=opts)


def test_cleaning_and_empty(tc):
    src, dst, n = tcgen.rmat(11, 16, 3)
    s2 = np.concatenate([dst, src, np.arange(50, dtype=np.int32)])
    d2 = np.concatenate([src, dst, np.arange(50, dtype=np.int32)])
    check_full(tc, s2, d2, n + 10)
    e = np.zeros(0, np.int32)
    with tc.build_csr(dev(np.array([0], np.int32)), dev(np.array([1], np.int32)), 2) as g:
        assert g.support().cpu().tolist() == [0]
    with tc.build_csr(dev(e), dev(e), 0) as g:
        assert g.m == 0 and g.support().numel() == 0


def test_c5_lattice_full(tc):
    """C5 at full size (30M edges, most supports 0 or 1): every edge bit-exact."""
    src, dst, n = tcgen.CONFIGS["C5"].generate(1)
    check_full(tc, src, dst, n)


@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_full_size_sampled(tc, cfg):
    """C2 / C3 at BASELINE size with the bench's launch configuration: 20,000
    sampled edges against the oracle one by one, and sum = 3T (stored oracle T)."""
    import json, os
    src, dst, n = tcgen.CONFIGS[cfg].generate(1)
    stored = json.load(open(os.path.join(os.path.dirname(__file__), "golden",
                                         "config_counts.json")))[f"{cfg}/seed1"]
    with tc.build_csr(dev(src), dev(dst), n) as g:
        sup = g.support()
        total = int(sup.to(torch.int64).sum().item())  # values < 2^31: int32 view is exact
        idx = torch.randint(0, g.m, (20000,), generator=torch.Generator().manual_seed(5)).cuda()
        u, v = g.edge_list()
        su, sv, ss = (x[idx].cpu().numpy() for x in (u, v, sup))
        assert g.m == stored["m"]
    assert total == 3 * stored["triangles"]
    og = oracle.SupportGraph(src, dst, n)
    want = og.pairs(su, sv)
    og.close()
    assert (want >= 0).all()  # every GPU edge is an edge of the cleaned input
    assert np.array_equal(ss.view(np.uint32).astype(np.int64), want)
