"""Test-side graph families with closed-form triangle counts, and brute-force
counters that share nothing with either the oracle or the CUDA path.

Closed forms (SURVEY.md §4.2 / §8(c) "What pins each part"):
  K_n -> C(n,3);  K_{a,b} and every bipartite graph (trees, stars, paths,
  even cycles, grids, hypercubes) -> 0;  C_3 -> 1, C_n (n >= 4) -> 0;
  Petersen -> 0 (girth 5);  wheel W_k (hub + k-cycle, k >= 4) -> k;
  friendship F_k -> k;  complete 3-partite K_{a,b,c} -> a*b*c.
"""
from __future__ import annotations

import itertools
from math import comb

import numpy as np


def _arr(edges, n):
    e = np.array(list(edges), dtype=np.int64).reshape(-1, 2)
    return e[:, 0].astype(np.int32), e[:, 1].astype(np.int32), n


def complete(n):
    return _arr(itertools.combinations(range(n), 2), n), comb(n, 3)


def complete_bipartite(a, b):
    return _arr(((i, a + j) for i in range(a) for j in range(b)), a + b), 0


def complete_multipartite(*sizes):
    starts = np.cumsum((0,) + sizes)
    parts = [range(starts[i], starts[i + 1]) for i in range(len(sizes))]
    edges = [(x, y) for p, q in itertools.combinations(parts, 2) for x in p for y in q]
    t = sum(a * b * c for a, b, c in itertools.combinations(sizes, 3))
    return _arr(edges, int(starts[-1])), t


def path(n):
    return _arr(((i, i + 1) for i in range(n - 1)), n), 0


def cycle(n):
    return _arr(((i, (i + 1) % n) for i in range(n)), n), 1 if n == 3 else 0


def star(k):
    return _arr(((0, i) for i in range(1, k + 1)), k + 1), 0


def grid(r, c):
    edges = []
    for i in range(r):
        for j in range(c):
            v = i * c + j
            if j + 1 < c:
                edges.append((v, v + 1))
            if i + 1 < r:
                edges.append((v, v + c))
    return _arr(edges, r * c), 0


def hypercube(d):
    n = 1 << d
    return _arr(((v, v ^ (1 << b)) for v in range(n) for b in range(d) if v < v ^ (1 << b)), n), 0


def petersen():
    outer = [(i, (i + 1) % 5) for i in range(5)]
    spokes = [(i, i + 5) for i in range(5)]
    inner = [(5 + i, 5 + (i + 2) % 5) for i in range(5)]
    return _arr(outer + spokes + inner, 10), 0


def wheel(k):
    rim = [(1 + i, 1 + (i + 1) % k) for i in range(k)]
    return _arr([(0, 1 + i) for i in range(k)] + rim, k + 1), (k if k >= 4 else 4)


def friendship(k):
    edges = []
    for i in range(k):
        a, b = 1 + 2 * i, 2 + 2 * i
        edges += [(0, a), (0, b), (a, b)]
    return _arr(edges, 2 * k + 1), k


def random_tree(n, rng):
    parent = [int(rng.integers(0, i)) for i in range(1, n)]
    return _arr(((i + 1, p) for i, p in enumerate(parent)), n), 0


def closed_form_cases():
    rng = np.random.default_rng(7)
    cases = {}
    for n in (1, 2, 3, 4, 5, 6, 10, 17, 33, 64, 100):
        cases[f"K{n}"] = complete(n)
    cases["K7,9"] = complete_bipartite(7, 9)
    cases["K40,40"] = complete_bipartite(40, 40)
    cases["K3,4,5"] = complete_multipartite(3, 4, 5)
    cases["T(12,3)"] = complete_multipartite(4, 4, 4)
    cases["K5,6,7,8"] = complete_multipartite(5, 6, 7, 8)
    cases["path50"] = path(50)
    cases["C3"] = cycle(3)
    cases["C9"] = cycle(9)
    cases["star20"] = star(20)
    cases["star1000"] = star(1000)
    cases["grid10x10"] = grid(10, 10)
    cases["Q4"] = hypercube(4)
    cases["Q10"] = hypercube(10)
    cases["petersen"] = petersen()
    cases["W10"] = wheel(10)
    cases["W4"] = wheel(4)
    cases["F5"] = friendship(5)
    cases["F300"] = friendship(300)
    cases["tree500"] = random_tree(500, rng)
    return cases


# ---------------------------------------------------------------- brute force

def dense_adjacency(src, dst, n):
    """0/1 symmetric adjacency of the cleaned simple graph (weights ignored)."""
    A = np.zeros((n, n), dtype=np.int64)
    A[src, dst] = 1
    A[dst, src] = 1
    np.fill_diagonal(A, 0)
    return A


def brute_force_triples(src, dst, n):
    """O(n^3) enumeration of vertex triples (the definition of T)."""
    A = dense_adjacency(src, dst, n)
    return sum(1 for x, y, z in itertools.combinations(range(n), 3)
               if A[x, y] and A[y, z] and A[x, z])


def trace_a3(src, dst, n):
    """trace(A^3) / 6: closed walks of length 3."""
    A = dense_adjacency(src, dst, n)
    return int(np.trace(A @ A @ A)) // 6


def lu_hadamard(src, dst, n):
    """B = L.U, C = A o B, T = sum(C) / 2."""
    A = dense_adjacency(src, dst, n)
    L, U = np.tril(A, -1), np.triu(A, 1)
    return int((A * (L @ U)).sum()) // 2


def sparse_trace(src, dst, n):
    """sum(A o A^2) / 6 with scipy sparse 0/1 matrices (medium graphs)."""
    import scipy.sparse as sp
    keep = src != dst
    s, d = src[keep].astype(np.int64), dst[keep].astype(np.int64)
    A = sp.coo_matrix((np.ones(len(s) * 2, dtype=np.int64),
                       (np.concatenate([s, d]), np.concatenate([d, s]))), shape=(n, n)).tocsr()
    A.data[:] = 1  # duplicates summed -> back to 0/1
    A.sum_duplicates()
    A.data[:] = 1
    return int((A @ A).multiply(A).sum()) // 6


def unique_undirected(src, dst):
    s, d = np.minimum(src, dst).astype(np.int64), np.maximum(src, dst).astype(np.int64)
    keep = s != d
    return np.unique(s[keep] << 32 | d[keep])
