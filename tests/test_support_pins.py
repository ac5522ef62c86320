"""Pins for the oracle's per-edge support (-m "not gpu").

sup(a,b) = number of triangles containing the edge {a,b}.  The oracle
(tco_support_* in oracle/tc_oracle.cpp) computes |N(a) ∩ N(b)|; it is pinned
here against closed forms, the matrix identity sup = (A·A)[a,b] for edges
(dense brute force and scipy sparse), triple enumeration, sum = 3T, and the
P:287 cleaning invariance.
"""
import itertools

import numpy as np
import pytest

import oracle
import tcgen
from tests import graphs


def as_dict(a, b, s):
    return {(int(x), int(y)): int(z) for x, y, z in zip(a, b, s)}


def test_complete_graph_every_edge_in_n_minus_2():
    for n in (3, 4, 7, 25):
        (src, dst, _), _ = graphs.complete(n)
        a, b, s = oracle.support(src, dst, n)
        assert len(s) == n * (n - 1) // 2
        assert (s == n - 2).all()


def test_wheel_spokes_and_rim():
    """W_k (hub 0 + k-cycle rim, k >= 4): a spoke lies in 2 triangles, a rim edge in 1."""
    k = 9
    (src, dst, n), _ = graphs.wheel(k)
    sup = as_dict(*oracle.support(src, dst, n))
    for (x, y), c in sup.items():
        assert c == (2 if x == 0 else 1), (x, y, c)


def test_friendship_and_bipartite():
    (src, dst, n), _ = graphs.friendship(12)
    assert (oracle.support(src, dst, n)[2] == 1).all()
    (src, dst, n), _ = graphs.complete_bipartite(6, 9)
    a, b, s = oracle.support(src, dst, n)
    assert len(s) == 54 and (s == 0).all()


def test_complete_tripartite_edge_sees_the_third_part():
    sizes = (3, 4, 5)
    (src, dst, n), _ = graphs.complete_multipartite(*sizes)
    part = np.repeat(np.arange(3), sizes)
    for (x, y), c in as_dict(*oracle.support(src, dst, n)).items():
        third = 3 - part[x] - part[y]
        assert c == sizes[third]


def test_edge_order_and_canonical_pairs():
    src = np.array([5, 1, 2, 2, 0, 3, 1], np.int32)
    dst = np.array([1, 5, 0, 2, 1, 4, 2], np.int32)
    a, b, s = oracle.support(src, dst, 6)
    assert list(zip(a.tolist(), b.tolist())) == [(0, 1), (0, 2), (1, 2), (1, 5), (3, 4)]
    assert s.tolist() == [1, 1, 1, 0, 0]


@pytest.mark.parametrize("seed", range(8))
def test_random_tiny_vs_dense_a_squared(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(3, 30))
    A = np.triu(rng.random((n, n)) < rng.uniform(0.1, 0.8), 1)
    src, dst = (x.astype(np.int32) for x in np.nonzero(A))
    D = graphs.dense_adjacency(src, dst, n)
    A2 = D @ D
    a, b, s = oracle.support(src, dst, n)
    assert len(s) == int(D.sum()) // 2
    for x, y, c in zip(a, b, s):
        assert D[x, y] == 1 and c == A2[x, y]
        # triple enumeration: w closes a triangle with {x, y}
        assert c == sum(1 for w in range(n) if D[x, w] and D[y, w])


@pytest.mark.parametrize("name,n", [("karate.txt", 34), ("lesmis.txt", 77)])
def test_golden_graphs_sum_is_three_t(golden, name, n):
    src, dst = golden(name)
    a, b, s = oracle.support(src, dst, n)
    assert int(s.sum()) == 3 * graphs.trace_a3(src, dst, n)
    D = graphs.dense_adjacency(src, dst, n)
    assert (s == (D @ D)[a, b]).all()


@pytest.mark.parametrize("scale,ef,seed", [(10, 16, 1), (12, 8, 4)])
def test_rmat_vs_sparse_a_squared(scale, ef, seed):
    import scipy.sparse as sp
    src, dst, n = tcgen.rmat(scale, ef, seed)
    a, b, s = oracle.support(src, dst, n)
    keys = graphs.unique_undirected(src, dst)
    assert np.array_equal((a.astype(np.int64) << 32) | b, keys)
    ka, kb = keys >> 32, keys & 0xFFFFFFFF
    A = sp.coo_matrix((np.ones(2 * len(keys), np.int64),
                       (np.concatenate([ka, kb]), np.concatenate([kb, ka]))), shape=(n, n)).tocsr()
    A2 = (A @ A).tocsr()
    assert np.array_equal(np.asarray(A2[ka, kb]).ravel(), s.astype(np.int64))
    assert int(s.sum()) == 3 * graphs.sparse_trace(src, dst, n)


def test_cleaning_invariance():
    rng = np.random.default_rng(3)
    src, dst, n = tcgen.rmat(10, 16, 7)
    base = oracle.support(src, dst, n)
    dup = rng.integers(0, len(src), 2000)
    loops = rng.integers(0, n, 100).astype(np.int32)
    s2 = np.concatenate([dst[dup], src, loops]).astype(np.int32)
    d2 = np.concatenate([src[dup], dst, loops]).astype(np.int32)
    got = oracle.support(s2, d2, n + 50)
    for x, y in zip(base, got):
        assert np.array_equal(x, y)


def test_pairs_matches_all_and_rejects_non_edges():
    src, dst, n = tcgen.rmat(10, 16, 2)
    g = oracle.SupportGraph(src, dst, n)
    a, b, s = g.all()
    idx = np.random.default_rng(0).integers(0, len(s), 300)
    assert np.array_equal(g.pairs(a[idx], b[idx]), s[idx].astype(np.int64))
    assert np.array_equal(g.pairs(b[idx], a[idx]), s[idx].astype(np.int64))  # order-free
    present = set(zip(a.tolist(), b.tolist()))
    non = [(x, y) for x, y in itertools.combinations(range(40), 2) if (x, y) not in present][:50]
    xa, xb = np.array(non, np.int32).T
    assert (g.pairs(xa, xb) == -1).all()
    assert (g.pairs(np.array([3], np.int32), np.array([3], np.int32)) == -1).all()
    g.close()


def test_degenerate_and_invalid():
    e = np.zeros(0, np.int32)
    a, b, s = oracle.support(e, e, 0)
    assert len(a) == len(b) == len(s) == 0
    with pytest.raises(ValueError):
        oracle.support(np.array([0, 7], np.int32), np.array([1, 2], np.int32), 5)
