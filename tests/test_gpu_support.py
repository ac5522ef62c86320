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


def stratified_positions(g, n_random=20000, n_hubs=64, per_hub=50, n_heads=2000, min_head_degree=0,
                         seed=5):
    """CSR positions to check one by one: edges of the n_hubs highest-degree
    vertices (up to per_hub each, in- and out-edges), one in-edge (a member of
    its group) and one out-edge (a table entry) of each of the n_heads heads v
    with the largest d+(v) (every head with d+(v) > min_head_degree when that
    is given: the global-probe "huge" groups of a low huge_degree), and
    n_random uniform positions."""
    rp, col, _ = g.csr()
    m = g.m
    gen = torch.Generator(device="cuda").manual_seed(seed)
    dplus = rp[1:] - rp[:-1]
    dminus = torch.bincount(col.long(), minlength=g.n)
    deg = dplus + dminus
    picks = [torch.randint(0, m, (n_random,), device="cuda", generator=gen)]
    hubs = torch.topk(deg, min(n_hubs, g.n)).indices
    heads = (torch.nonzero(dplus > min_head_degree).flatten() if min_head_degree
             else torch.topk(dplus, min(n_heads, g.n)).indices)
    # in-edges (u, x) of x in hubs / heads: positions where col == x
    for verts, cap in ((hubs, per_hub), (heads, 1)):
        mark = torch.zeros(g.n, dtype=torch.bool, device="cuda")
        mark[verts] = True
        pos = torch.nonzero(mark[col.long()]).flatten()
        if pos.numel():
            key = col.long()[pos] * (m + 1) + torch.randint(0, m, (pos.numel(),), device="cuda",
                                                          generator=gen)
            pos = pos[torch.argsort(key)]
            c = col.long()[pos]
            first = torch.ones_like(c, dtype=torch.bool)
            first[1:] = c[1:] != c[:-1]
            start = torch.nonzero(first).flatten()
            rank_in = torch.arange(pos.numel(), device="cuda") - start[torch.cumsum(first.long(), 0) - 1]
            picks.append(pos[rank_in < cap])
        # out-edges of x: positions rp[x] .. rp[x] + min(d+, cap)
        lo, d = rp[verts], dplus[verts]
        k = torch.arange(cap, device="cuda")
        outp = (lo[:, None] + k[None, :])[(k[None, :] < d[:, None])]
        picks.append(outp)
    return torch.unique(torch.cat(picks))


def check_positions(g, sup, idx, src, dst, n):
    u, v = g.edge_list()
    su, sv, ss = (x[idx].cpu().numpy() for x in (u, v, sup))
    og = oracle.SupportGraph(src, dst, n)
    want = og.pairs(su, sv)
    og.close()
    assert (want >= 0).all()  # every GPU edge is an edge of the cleaned input
    bad = np.nonzero(ss.view(np.uint32).astype(np.int64) != want)[0]
    assert bad.size == 0, f"{bad.size} of {len(idx)} edges differ, e.g. {su[bad[:5]]}-{sv[bad[:5]]}"


@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_full_size_stratified(tc, cfg):
    """C2 / C3 at BASELINE size with the bench's launch configuration: sum = 3T
    (the oracle's stored T), and against the oracle one by one the edges of the
    64 highest-degree vertices, an in- and an out-edge of the 2,000 heads with
    the largest tables, and 20,000 uniform edges.  Then the same graph with
    huge_degree = 256, so every head with d+(v) > 256 is probed in global
    memory (32 at C2, whose max d+ is ~100): one in- and one out-edge of each.""" 
    import json, os
    src, dst, n = tcgen.CONFIGS[cfg].generate(1)
    stored = json.load(open(os.path.join(os.path.dirname(__file__), "golden",
                                         "config_counts.json")))[f"{cfg}/seed1"]
    with tc.build_csr(dev(src), dev(dst), n) as g:
        assert g.m == stored["m"]
        sup = g.support()
        assert int(sup.to(torch.int64).sum().item()) == 3 * stored["triangles"]
        idx = stratified_positions(g)
        check_positions(g, sup, idx, src, dst, n)
    hd = {"C2": 32, "C3": 256}[cfg]
    with tc.build_csr(dev(src), dev(dst), n, options={"huge_degree": hd}) as g:
        sup = g.support()
        assert int(sup.to(torch.int64).sum().item()) == 3 * stored["triangles"]
        idx = stratified_positions(g, n_random=2000, n_hubs=16, per_hub=8, min_head_degree=hd)
        assert idx.numel() > 4000
        check_positions(g, sup, idx, src, dst, n)
