"""Pins for the CPU oracle (-m "not gpu").

The oracle (oracle/tc_oracle.cpp) is checked against things that do NOT come
from itself: closed forms, a published count (karate = 45), the paper's worked
examples, brute force / linear-algebra identities and
invariances the paper asserts.  A dropped term, an off-by-one in the
orientation or a double count fails at least one of these.
"""
from math import comb

import numpy as np
import pytest

import oracle
import tcgen
from tests import graphs


@pytest.mark.parametrize("name", sorted(graphs.closed_form_cases()))
def test_closed_forms(name):
    (src, dst, n), t = graphs.closed_form_cases()[name]
    assert oracle.triangles(src, dst, n) == t


def test_fig1b_worked_example():
    """PAPER.md P:78 (Fig. 1(b)): N(2) = {1,3,4,5}, N(5) = {0,2,4}; wSet of edge
    (2,5) is {4}.  The graph made of exactly those two neighbourhoods has the
    single triangle {2,4,5}."""
    edges = [(2, 1), (2, 3), (2, 4), (2, 5), (5, 0), (5, 2), (5, 4)]
    src, dst = np.array(edges, dtype=np.int32).T
    assert oracle.triangles(src, dst, 6) == 1


def test_karate_published(golden):
    src, dst = golden("karate.txt")
    r = oracle.count(src, dst, 34)
    assert r.triangles == 45
    assert r.m == 78 and r.n_active == 34


@pytest.mark.parametrize("name,n", [("lesmis.txt", 77), ("florentine.txt", 15), ("davis.txt", 32)])
def test_real_graphs_brute_force(golden, name, n):
    src, dst = golden(name)
    t = oracle.triangles(src, dst, n)
    assert t == graphs.trace_a3(src, dst, n) == graphs.lu_hadamard(src, dst, n)
    if name == "davis.txt":
        assert t == 0  # bipartite
    if name == "florentine.txt":
        assert t == 3


@pytest.mark.parametrize("seed", range(12))
def test_random_tiny_brute_force(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(3, 28))
    p = float(rng.uniform(0.05, 0.9))
    A = np.triu(rng.random((n, n)) < p, 1)
    src, dst = np.nonzero(A)
    src, dst = src.astype(np.int32), dst.astype(np.int32)
    t = oracle.triangles(src, dst, n)
    assert t == graphs.brute_force_triples(src, dst, n)
    assert t == graphs.trace_a3(src, dst, n)
    assert t == graphs.lu_hadamard(src, dst, n)


@pytest.mark.parametrize("scale,ef,seed", [(8, 8, 1), (10, 16, 2), (12, 16, 3), (11, 4, 4)])
def test_rmat_vs_sparse_trace(scale, ef, seed):
    src, dst, n = tcgen.rmat(scale, ef, seed)
    r = oracle.count(src, dst, n)
    assert r.triangles == graphs.sparse_trace(src, dst, n)
    assert r.m == len(graphs.unique_undirected(src, dst))
    # degree orientation bounds the out-degree by sqrt(2m)
    assert r.max_out_degree <= int(np.sqrt(2 * r.m))


def test_networkx_powerlaw_cluster():
    nx = pytest.importorskip("networkx")
    G = nx.powerlaw_cluster_graph(400, 5, 0.5, seed=3)
    e = np.array(G.edges(), dtype=np.int32)
    t = sum(nx.triangles(G).values()) // 3
    assert oracle.triangles(e[:, 0], e[:, 1], 400) == t


def test_orientation_independence():
    """C-3: any total order counts each triangle once (id / degree / hashed)."""
    src, dst, n = tcgen.rmat(12, 16, 9)
    ts = {oracle.triangles(src, dst, n, order=o) for o in (0, 1, 2)}
    assert len(ts) == 1


def test_cleaning_invariance():
    """removing isolated vertices, self-loops and duplicates does not
    alter T — so injecting them must not change the oracle's count."""
    rng = np.random.default_rng(5)
    src, dst, n = tcgen.rmat(11, 16, 5)
    base = oracle.count(src, dst, n)
    dup = rng.integers(0, len(src), 5000)
    loops = rng.integers(0, n, 300).astype(np.int32)
    s2 = np.concatenate([src, dst[dup], loops, src[dup]]).astype(np.int32)
    d2 = np.concatenate([dst, src[dup], loops, dst[dup]]).astype(np.int32)
    perm = rng.permutation(len(s2))
    r = oracle.count(s2[perm], d2[perm], n + 5000)  # 5000 extra isolated vertices
    assert r.triangles == base.triangles and r.m == base.m and r.n_active == base.n_active


def test_relabel_invariance():
    rng = np.random.default_rng(11)
    src, dst, n = tcgen.rmat(11, 8, 6)
    p = rng.permutation(n).astype(np.int32)
    assert oracle.triangles(p[src], p[dst], n) == oracle.triangles(src, dst, n)


def test_disjoint_union_additive():
    s1, d1, n1 = tcgen.rmat(10, 16, 1)
    s2, d2, n2 = tcgen.lattice(40, 2)
    t1, t2 = oracle.triangles(s1, d1, n1), oracle.triangles(s2, d2, n2)
    s = np.concatenate([s1, s2 + n1]).astype(np.int32)
    d = np.concatenate([d1, d2 + n1]).astype(np.int32)
    assert oracle.triangles(s, d, n1 + n2) == t1 + t2


def test_degenerate_inputs():
    e = np.zeros(0, dtype=np.int32)
    assert oracle.triangles(e, e, 0) == 0
    assert oracle.triangles(e, e, 10) == 0
    assert oracle.triangles(np.array([0], np.int32), np.array([1], np.int32), 2) == 0
    assert oracle.triangles(np.array([0, 1, 2], np.int32), np.array([1, 2, 0], np.int32), 3) == 1
    loops = np.arange(10, dtype=np.int32)
    r = oracle.count(loops, loops, 10)
    assert r.triangles == 0 and r.m == 0 and r.n_active == 0


def test_invalid_ids_rejected():
    with pytest.raises(ValueError):
        oracle.count(np.array([0, 5], np.int32), np.array([1, 2], np.int32), 5)
    with pytest.raises(ValueError):
        oracle.count(np.array([-1], np.int32), np.array([1], np.int32), 5)


def test_sampling_partitions_rows():
    """sample_stride only restricts which rows are counted; the bench scales by
    merge steps, so the counted steps must add up over the strides' cosets."""
    src, dst, n = tcgen.rmat(12, 16, 3)
    full = oracle.count(src, dst, n)
    s = oracle.count(src, dst, n, sample_stride=4)
    assert s.merge_steps_total == full.merge_steps_total
    assert 0 < s.merge_steps_counted < full.merge_steps_total
    assert s.triangles <= full.triangles


@pytest.mark.slow
def test_k3000_exceeds_32_bits():
    """C-13: C(3000,3) = 4,495,501,000 > 2^32 catches a 32-bit accumulator."""
    (src, dst, n), t = graphs.complete(3000)
    assert t == comb(3000, 3) > 2**32
    assert oracle.triangles(src, dst, n) == t


def test_sample_offsets_tile_the_rows():
    """count_rows over the cosets x % s == o, o = 0..s-1, adds up to the full count."""
    src, dst, n = tcgen.rmat(12, 16, 13)
    g = oracle.OracleGraph(src, dst, n)
    full = g.count_rows()
    parts = [g.count_rows(stride=5, offset=o) for o in range(5)]
    assert sum(p.triangles for p in parts) == full.triangles == oracle.triangles(src, dst, n)
    assert sum(p.merge_steps_counted for p in parts) == full.merge_steps_total
