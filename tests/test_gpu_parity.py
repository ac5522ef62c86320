"""GPU parity: the CUDA path (through the C-ABI) vs the CPU oracle, bit-exact.

Every count here is compared with oracle/ (or a closed form) on the same
seeded input from tcgen/; neither side's numbers come from the other.
Sizes span many work chunks and ragged tails; the plan options are varied
because they must never change a count.
"""
import os
from math import comb

import numpy as np
import pytest

import oracle
import tcgen
from tests import graphs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

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


def gpu_count(tc, src, dst, n=None, **kw):
    with tc.build_csr(dev(src), dev(dst), n, **kw) as g:
        return g.count()


# ------------------------------------------------------------------ closed forms / golden

@pytest.mark.parametrize("name", sorted(graphs.closed_form_cases()))
def test_closed_forms(tc, name):
    (src, dst, n), t = graphs.closed_form_cases()[name]
    assert gpu_count(tc, src, dst, n) == t
    assert gpu_count(tc, src, dst, n, options={"long_min": 32}) == t  # with the long class


def test_karate(tc, golden):
    src, dst = golden("karate.txt")
    assert gpu_count(tc, src, dst, 34) == 45


@pytest.mark.parametrize("name", ["lesmis.txt", "florentine.txt", "davis.txt"])
def test_golden_vs_oracle(tc, golden, name):
    src, dst = golden(name)
    assert gpu_count(tc, src, dst) == oracle.triangles(src, dst)


def test_fig14_suffix_example(tc):
    """P:359 (Fig. 14): N(0) ⊇ {4,5,8}; edge (0,8) has an empty suffix and is
    skipped; edge (0,4) searches only [5,8].  Graph: 0-{4,5,8}, 4-{5,8}, 5-8
    is K4 on {0,4,5,8} plus nothing else -> 4 triangles."""
    e = np.array([(0, 4), (0, 5), (0, 8), (4, 5), (4, 8), (5, 8)], dtype=np.int32)
    assert gpu_count(tc, e[:, 0], e[:, 1], 9) == 4


# ------------------------------------------------------------------ configs

@pytest.mark.parametrize("seed", [1, 2, 3, 4, 5])
def test_c1_rmat10_seeds(tc, seed):
    src, dst, n = tcgen.CONFIGS["C1"].generate(seed)
    r = oracle.count(src, dst, n)
    assert gpu_count(tc, src, dst, n, options={"long_min": 32}) == r.triangles
    with tc.build_csr(dev(src), dev(dst), n) as g:
        assert g.count() == r.triangles
        assert g.m == r.m and g.n == r.n_active
        assert g.info.max_out_degree == r.max_out_degree  # same (deg, id) order


@pytest.mark.parametrize("scale,ef,seed", [(14, 16, 1), (16, 16, 2), (17, 8, 3)])
def test_rmat_medium(tc, scale, ef, seed):
    src, dst, n = tcgen.rmat(scale, ef, seed)
    assert gpu_count(tc, src, dst, n) == oracle.triangles(src, dst, n)


def test_rmat_skewed_initiator(tc):
    src, dst, n = tcgen.rmat(16, 24, 7, abc=(0.65, 0.15, 0.15))
    assert gpu_count(tc, src, dst, n) == oracle.triangles(src, dst, n)


def test_c2_chung_lu_full(tc):
    src, dst, n = tcgen.CONFIGS["C2"].generate(1)
    assert gpu_count(tc, src, dst, n) == oracle.triangles(src, dst, n)


def test_c5_lattice_full(tc):
    src, dst, n = tcgen.CONFIGS["C5"].generate(1)
    assert gpu_count(tc, src, dst, n) == oracle.triangles(src, dst, n)


@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_full_size_vs_stored_oracle(tc, cfg):
    """C3 (260M edges) and C4 (1.57B edges, the 8-GPU config, here on one GPU)
    at BASELINE size and in bench.py's launch configuration, against the
    oracle's exact count stored by tests/golden/make_config_counts.py (the
    input is regenerated and its checksum must match the stored one)."""
    import json, os
    stored = json.load(open(os.path.join(os.path.dirname(__file__), "golden",
                                         "config_counts.json")))[f"{cfg}/seed1"]
    src, dst, n = tcgen.CONFIGS[cfg].generate(1)
    assert tcgen.checksum(src, dst) == stored["checksum"]
    ds, dd = dev(src), dev(dst)
    del src, dst
    with tc.build_csr(ds, dd, n) as g:
        del ds, dd
        assert g.m == stored["m"] and g.n == stored["n_active"]
        assert g.info.max_out_degree == stored["max_out_degree"]
        assert g.count() == stored["triangles"]
        b = g.partition(8)  # the 8-rank split of the multi-GPU run, emulated on one GPU
        parts = [int(g.count_range(b[r], b[r + 1]).item()) for r in range(8)]
        assert sum(parts) == stored["triangles"]


def test_chung_lu_small(tc):
    src, dst, n = tcgen.chung_lu(200_000, 1_500_000, 3)
    assert gpu_count(tc, src, dst, n) == oracle.triangles(src, dst, n)


# ------------------------------------------------------------------ properties

@pytest.mark.parametrize("opts", [
    dict(chunk_cost=64), dict(chunk_cost=256), dict(chunk_cost=4096), dict(chunk_cost=1 << 20),
    dict(block_threads=64), dict(block_threads=128), dict(block_threads=256),
    dict(block_threads=512), dict(block_threads=96),
    dict(seg_cost=1), dict(seg_cost=64), dict(table_factor=2), dict(table_factor=16),
    dict(huge_degree=1), dict(huge_degree=16), dict(huge_degree=16, chunk_cost=64),
    dict(long_min=1), dict(long_min=8), dict(long_min=1 << 30), dict(long_min=1 << 30, chunk_cost=64),
    dict(probe_mode=1), dict(probe_mode=1, long_min=1), dict(probe_mode=1, long_min=1 << 30),
    dict(table_factor=2, chunk_cost=1 << 20),
    dict(bitmap_factor=-1), dict(bitmap_factor=1), dict(bitmap_factor=64),
    dict(bitmap_factor=64, probe_mode=1), dict(bitmap_factor=64, long_min=1 << 30),
    dict(bitmap_factor=-1, long_min=1),
    # explicit long_min = 32: the two-class split large graphs use (a graph this
    # small is otherwise all short class)
    dict(long_min=32), dict(long_min=32, chunk_cost=64), dict(long_min=32, block_threads=128),
    dict(long_min=32, probe_mode=1), dict(long_min=32, bitmap_factor=-1),
    dict(long_min=32, table_factor=2), dict(long_min=32, huge_degree=16),
    dict(long_min=32, bitmap_factor=64),
])
def test_plan_options_never_change_count(tc, opts):
    src, dst, n = tcgen.rmat(13, 16, 11)
    t = oracle.triangles(src, dst, n)
    with tc.build_csr(dev(src), dev(dst), n, options=opts) as g:
        assert g.count() == t
    with tc.build_csr(dev(src), dev(dst), n) as g:
        g.replan(opts)
        assert g.count() == t


def test_cleaning_invariance(tc):
    """duplicates, reversed pairs, self-loops, isolated vertices."""
    rng = np.random.default_rng(5)
    src, dst, n = tcgen.rmat(12, 16, 5)
    base = gpu_count(tc, src, dst, n)
    dup = rng.integers(0, len(src), 20000)
    loops = rng.integers(0, n, 500).astype(np.int32)
    s2 = np.concatenate([src, dst[dup], loops, src[dup]])
    d2 = np.concatenate([dst, src[dup], loops, dst[dup]])
    p = rng.permutation(len(s2))
    assert gpu_count(tc, s2[p], d2[p], n + 1000) == base
    assert gpu_count(tc, s2[p], d2[p], n + 1000, keep_isolated=True) == base


def test_relabel_invariance(tc):
    rng = np.random.default_rng(2)
    src, dst, n = tcgen.rmat(13, 8, 2)
    perm = rng.permutation(n).astype(np.int32)
    assert gpu_count(tc, perm[src], perm[dst], n) == gpu_count(tc, src, dst, n)


def test_disjoint_union_additive(tc):
    s1, d1, n1 = tcgen.rmat(11, 16, 1)
    s2, d2, n2 = tcgen.lattice(60, 2)
    s = np.concatenate([s1, s2 + n1])
    d = np.concatenate([d1, d2 + n1])
    assert gpu_count(tc, s, d) == gpu_count(tc, s1, d1) + gpu_count(tc, s2, d2)


@pytest.mark.parametrize("world", [1, 2, 3, 5, 8])
def test_partition_ranges_sum_to_total(tc, world):
    src, dst, n = tcgen.rmat(14, 16, 4)
    t = oracle.triangles(src, dst, n)
    with tc.build_csr(dev(src), dev(dst), n, options=dict(chunk_cost=2048)) as g:
        b = g.partition(world)
        assert b[0] == 0 and b[-1] == g.m_live and b == sorted(b)
        parts = [int(g.count_range(b[r], b[r + 1]).item()) for r in range(world)]
        assert sum(parts) == t


def test_arbitrary_ranges_sum_to_total(tc):
    """Any cut of [0, m_live) is exact, including cuts inside chunks."""
    rng = np.random.default_rng(9)
    src, dst, n = tcgen.rmat(13, 16, 8)
    t = oracle.triangles(src, dst, n)
    with tc.build_csr(dev(src), dev(dst), n, options=dict(chunk_cost=1024)) as g:
        cuts = np.unique(np.concatenate([[0, g.m_live], rng.integers(0, g.m_live, 37)]))
        parts = [int(g.count_range(a, b).item()) for a, b in zip(cuts, cuts[1:])]
        assert sum(parts) == t
        assert int(g.count_range(5, 5).item()) == 0


def test_count_async_matches(tc):
    src, dst, n = tcgen.rmat(12, 16, 3)
    with tc.build_csr(dev(src), dev(dst), n) as g:
        out = g.count_async()
        torch.cuda.synchronize()
        assert int(out.item()) == g.count() == oracle.triangles(src, dst, n)


def test_host_entry_point(tc):
    src, dst, n = tcgen.rmat(12, 16, 6)
    with tc.build_csr_host(src, dst, n) as g:
        assert g.count() == oracle.triangles(src, dst, n)
    pinned_s = torch.from_numpy(src).pin_memory()
    pinned_d = torch.from_numpy(dst).pin_memory()
    with tc.build_csr_host(pinned_s, pinned_d, n) as g:
        assert g.count() == oracle.triangles(src, dst, n)


# ------------------------------------------------------------------ CSR layout

def reference_csr(src, dst, n):
    """Host reference of a1..a5 (numpy): (deg, id) rank, relabel, orient, sort."""
    s = np.minimum(src, dst).astype(np.int64)
    d = np.maximum(src, dst).astype(np.int64)
    keep = s != d
    key = np.unique((s[keep] << 32) | d[keep])
    a, b = key >> 32, key & 0xFFFFFFFF
    deg = np.bincount(np.concatenate([a, b]), minlength=n)
    active = np.nonzero(deg > 0)[0]
    order = active[np.lexsort((active, deg[active]))]
    rank = np.full(n, -1, dtype=np.int64)
    rank[order] = np.arange(len(order))
    u, v = rank[a], rank[b]
    lo, hi = np.minimum(u, v), np.maximum(u, v)
    idx = np.lexsort((hi, lo))
    lo, hi = lo[idx], hi[idx]
    row_ptr = np.concatenate([[0], np.cumsum(np.bincount(lo, minlength=len(order)))])
    return row_ptr, hi.astype(np.int32), order.astype(np.int32)


@pytest.mark.parametrize("case", ["rmat", "lattice", "karate", "dups"])
def test_csr_exact(tc, golden, case):
    if case == "rmat":
        src, dst, n = tcgen.rmat(12, 16, 2)
    elif case == "dups":  # every pair 3x, half reversed, plus self-loops: a2's dedup
        s0, d0, n = tcgen.rmat(14, 8, 4)
        src = np.concatenate([s0, d0, s0, np.arange(0, n, 7, dtype=np.int32)])
        dst = np.concatenate([d0, s0, d0, np.arange(0, n, 7, dtype=np.int32)])
    elif case == "lattice":
        src, dst, n = tcgen.lattice(50, 3)
    else:
        (src, dst), n = golden("karate.txt"), 34
    rp, col, perm = reference_csr(src, dst, n)
    with tc.build_csr(dev(src), dev(dst), n) as g:
        grp, gcol, gperm = (x.cpu().numpy() for x in g.csr())
        np.testing.assert_array_equal(grp, rp)
        np.testing.assert_array_equal(gcol, col)
        np.testing.assert_array_equal(gperm, perm)
        # invariants: rows strictly ascending, col > row, d+ <= sqrt(2m)
        rows = np.repeat(np.arange(len(rp) - 1), np.diff(rp))
        assert np.all(gcol > rows)
        same = rows[1:] == rows[:-1]
        assert np.all(gcol[1:][same] > gcol[:-1][same])
        assert np.diff(rp).max() <= int(np.sqrt(2 * g.m))


# ------------------------------------------------------------------ edge cases / errors

def test_empty_and_tiny(tc):
    e = np.zeros(0, dtype=np.int32)
    assert gpu_count(tc, e, e, 0) == 0
    assert gpu_count(tc, e, e, 10) == 0
    assert gpu_count(tc, e, e) == 0
    assert gpu_count(tc, [0], [1], 2) == 0
    assert gpu_count(tc, [0, 1, 2], [1, 2, 0]) == 1
    loops = np.arange(10, dtype=np.int32)
    assert gpu_count(tc, loops, loops, 10) == 0


def test_invalid_ids(tc):
    with pytest.raises(tc.InvalidArgument):
        tc.build_csr(dev([0, 5]), dev([1, 2]), 5)
    with pytest.raises(tc.InvalidArgument):
        tc.build_csr(dev([-1]), dev([1]), 5)
    with pytest.raises(tc.InvalidArgument):
        tc.build_csr(dev([-1]), dev([1]))
    # the library is still usable afterwards
    assert gpu_count(tc, [0, 1, 2], [1, 2, 0]) == 1


def test_sparse_ids_large_n(tc):
    """n_vertices = 2^31-1 with a handful of sparse ids."""
    big = 2**31 - 2
    src = np.array([0, 1000, big, 0], dtype=np.int32)
    dst = np.array([1000, big, 0, 7], dtype=np.int32)
    assert gpu_count(tc, src, dst, 2**31 - 1) == 1


def test_k3000_exceeds_32_bits(tc):
    """C-13: C(3000,3) > 2^32 catches any 32-bit accumulator above the thread."""
    (src, dst, n), t = graphs.complete(3000)
    assert t == comb(3000, 3) > 2**32
    assert gpu_count(tc, src, dst, n) == t


def test_classes_partition_the_edges(tc):
    """long_min only moves edges between the two classes (C-10 analogue)."""
    src, dst, n = tcgen.rmat(14, 16, 12)
    t = oracle.triangles(src, dst, n)
    for lm in (1, 4, 32, 200, 1 << 30):
        with tc.build_csr(dev(src), dev(dst), n, options=dict(long_min=lm)) as g:
            assert g.count() == t, lm


def test_lattice_trim_drops_edges(tc):
    """C5-like lattice: trimming the suffix to [min N+(v), max N+(v)] leaves
    far fewer live edges than m, and the count is unchanged."""
    src, dst, n = tcgen.lattice(300, 4)
    with tc.build_csr(dev(src), dev(dst), n) as g:
        assert g.count() == oracle.triangles(src, dst, n)
        assert g.m_live < 0.5 * g.m


def test_huge_table_path_on_clique(tc):
    """K_1200 with huge_degree=100: most tables go through the global probe."""
    (src, dst, n), t = graphs.complete(1200)
    assert gpu_count(tc, src, dst, n, options=dict(huge_degree=100)) == t


# ------------------------------------------------------------------ f3: the paper's Polak / TRUST kernels

def variant_counts(tc, src, dst, n):
    with tc.build_csr(dev(src), dev(dst), n) as g:
        return {v: int(g.count_variant(v).item()) for v in ("polak", "trust")}, g.count()


@pytest.mark.parametrize("name", ["K3", "K10", "K100", "W10", "F300", "K5,6,7,8", "Q10", "star1000"])
def test_variants_closed_forms(tc, name):
    (src, dst, n), t = graphs.closed_form_cases()[name]
    got, grouped = variant_counts(tc, src, dst, n)
    assert got == {"polak": t, "trust": t} and grouped == t


@pytest.mark.parametrize("cfg_seed", [("C1", 1), ("C1", 2), ("rmat16", 3), ("skew15", 4), ("C5", 1)])
def test_variants_vs_oracle(tc, cfg_seed):
    name, seed = cfg_seed
    if name == "rmat16":
        src, dst, n = tcgen.rmat(16, 16, seed)
    elif name == "skew15":
        src, dst, n = tcgen.rmat(15, 24, seed, abc=(0.65, 0.15, 0.15))
    else:
        src, dst, n = tcgen.CONFIGS[name].generate(seed)
    want = oracle.triangles(src, dst, n)
    got, grouped = variant_counts(tc, src, dst, n)
    assert got == {"polak": want, "trust": want} and grouped == want


def test_trust_bucket_overflow_fallback(tc, monkeypatch):
    """TC_TRUST_CAP=1 makes almost every TRUST bucket overflow, so both the warp
    and the block kernels take the binary-search fallback; T must not change."""
    src, dst, n = tcgen.rmat(14, 16, 5)
    want = oracle.triangles(src, dst, n)
    monkeypatch.setenv("TC_TRUST_CAP", "1")
    with tc.build_csr(dev(src), dev(dst), n) as g:
        assert g.info.max_out_degree > 100  # the block path runs too
        assert int(g.count_variant("trust").item()) == want


def test_dedup_paths_agree(tc):
    """a2 by hashing and by radix sort + unique (forced with TC_DEDUP in child
    processes) build the same CSR and count."""
    import hashlib
    import subprocess
    import sys
    src, dst, n = tcgen.rmat(16, 16, 9)
    code = ("import sys, hashlib, numpy as np, torch; sys.path.insert(0, %r); import tcgen;"
            "import paper_conf_ipps_li0ptz24_b200 as tc;"
            "s, d, n = tcgen.rmat(16, 16, 9);"
            "g = tc.build_csr(torch.from_numpy(s).cuda(), torch.from_numpy(d).cuda(), n);"
            "h = hashlib.sha256(); [h.update(x.cpu().numpy().tobytes()) for x in g.csr()];"
            "print(h.hexdigest(), g.count())") % ROOT
    out = {}
    for mode, env_kv in (("sort", {"TC_DEDUP": "sort"}), ("hash", {"TC_DEDUP": "hash"})):
        env = dict(os.environ, **env_kv)
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                           timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        out[mode] = r.stdout.split()[-2:]
    assert out["sort"] == out["hash"]
    assert int(out["sort"][1]) == oracle.triangles(src, dst)


@pytest.mark.parametrize("scale,ef,seed", [(18, 16, 3), (20, 8, 4)])
def test_sort_paths_agree(tc, scale, ef, seed):
    """The build's 64-bit key sorts with the tuned onesweep policy (a2, a5)
    and with CUB's default policy (forced with TC_SORT=cub in a child process)
    build the same CSR, B_ITC and count.  Scale 18 sorts 36-bit keys in 5
    passes (the result lands in the second buffer), scale 20 in 5 / 6."""
    import subprocess
    import sys
    src, dst, n = tcgen.rmat(scale, ef, seed)
    assert len(src) >= (1 << 20)
    code = ("import sys, hashlib, numpy as np, torch; sys.path.insert(0, %r); import tcgen;"
            "import paper_conf_ipps_li0ptz24_b200 as tc;"
            "s, d, n = tcgen.rmat(%d, %d, %d);"
            "g = tc.build_csr(torch.from_numpy(s).cuda(), torch.from_numpy(d).cuda(), n);"
            "h = hashlib.sha256(); [h.update(x.cpu().numpy().tobytes()) for x in g.csr()];"
            "print(h.hexdigest(), g.info.b_itc, g.info.keys_total, g.count())") % (ROOT, scale, ef, seed)
    out = {}
    for mode, env_kv in (("own", {}), ("cub", {"TC_SORT": "cub"})):  # own = the tuned policy
        env = dict(os.environ, **env_kv)
        env.pop("TC_SORT", None) if mode == "own" else None
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                           timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        out[mode] = r.stdout.split()[-4:]
    assert out["own"] == out["cub"]
    assert int(out["own"][3]) == oracle.triangles(src, dst)


def test_host_pipelined_build_equals_device(tc):
    """Above 2^25 pairs tc_build_csr_host overlaps the H2D copy of piece i+1
    with the sort of piece i and merges the sorted runs: the graph must be
    the one tc_build_csr builds from device arrays."""
    src, dst, n = tcgen.rmat(21, 20, 6)  # 41.9 M pairs
    assert len(src) > (1 << 25)
    ps = torch.from_numpy(src).pin_memory()
    pd = torch.from_numpy(dst).pin_memory()
    with tc.build_csr(dev(src), dev(dst), n) as g0, tc.build_csr_host(ps, pd, n) as g1:
        for a, b in zip(g0.csr(), g1.csr()):
            assert torch.equal(a, b)
        assert g1.count() == g0.count()
        assert g1.info.b_itc == g0.info.b_itc


@pytest.mark.parametrize("n,opts", [
    (1500, dict(table_factor=16, bitmap_factor=-1, long_min=32)),   # 16 d+ > the cap -> load 1/3
    (3000, dict(table_factor=16, bitmap_factor=-1, long_min=32)),   # -> load 1/3 (long) and 1/2 (short)
    (3000, dict(table_factor=16, bitmap_factor=-1, long_min=1 << 30)),
])
def test_table_cap_fallbacks(tc, n, opts):
    """Hash tables that would exceed their class's SMEM cap at table_factor
    fall back to load 1/3, then 1/2, before going to global binary search;
    the count is unchanged (K_n: C(n, 3), > 2^32 at n = 3000)."""
    (src, dst, nn), t = graphs.complete(n)
    assert gpu_count(tc, src, dst, nn, options=opts) == t


def test_more_than_2_31_edges(tc):
    """m in [2^31, 2^32): every col index of the plan and the count kernel's
    32-bit tile descriptors passes 2^31 (the guard only rejects m >= 2^32).
    A disjoint union of c copies of K_64 with m = c * C(64, 2) > 2^31 unique
    edges, generated on the device; T = c * C(64, 3) in closed form (C-16)."""
    torch.cuda.empty_cache()
    tc.release_memory()  # the earlier tests' cached pool memory
    free, _ = torch.cuda.mem_get_info()
    if free < (170 << 30):
        pytest.skip(f"needs ~170 GB of device memory, {free >> 30} GB free")
    k = 64
    iu = torch.triu_indices(k, k, offset=1, device="cuda").to(torch.int32)  # C(64, 2) pairs
    c = (2**31) // iu.shape[1] + 4096
    m = c * iu.shape[1]
    assert 2**31 < m < 2**32
    off = (torch.arange(c, device="cuda", dtype=torch.int32) * k)[:, None]
    src = (off + iu[0][None, :]).reshape(-1)
    dst = (off + iu[1][None, :]).reshape(-1)
    del off
    with tc.build_csr(src, dst, c * k) as g:
        del src, dst
        assert g.m == m and g.n == c * k and g.info.max_out_degree == k - 1
        assert g.count() == c * comb(k, 3)
        b = g.partition(3)
        assert sum(int(g.count_range(b[r], b[r + 1]).item()) for r in range(3)) == c * comb(k, 3)


def test_close_waits_only_for_its_own_work(tc):
    """tc_free waits for the work other streams enqueued on the graph (the
    stream-ordered entry points record an event), not for the device: a graph
    closed right after an async count on another stream still yields T."""
    src, dst, n = tcgen.rmat(16, 16, 21)
    want = oracle.triangles(src, dst)
    s = torch.cuda.Stream()
    out = torch.zeros(1, dtype=torch.int64, device="cuda")
    g = tc.build_csr(dev(src), dev(dst), n)
    g.count_async(out=out, stream=s)
    g.close()
    junk = [torch.full((1 << 22,), -1, dtype=torch.int32, device="cuda") for _ in range(4)]
    s.synchronize()
    assert int(out.item()) == want
    del junk


def test_build_and_count_on_two_streams_concurrently(tc):
    """The pipelined use (bench.py e2e_pipelined): graph i+1 is built from
    host pairs on one stream in a second host thread while graph i is counted
    on another stream; every count equals the oracle's."""
    import threading
    src, dst, n = tcgen.rmat(17, 16, 22)
    want = oracle.triangles(src, dst)
    ps = torch.from_numpy(src).pin_memory()
    pd = torch.from_numpy(dst).pin_memory()
    sb, sc = torch.cuda.Stream(), torch.cuda.Stream()
    g = tc.build_csr_host(ps, pd, n, stream=sb)
    for _ in range(3):
        res = {}

        def build():
            with torch.cuda.stream(sb):
                res["g"] = tc.build_csr_host(ps, pd, n, stream=sb)

        th = threading.Thread(target=build)
        th.start()
        assert g.count(stream=sc) == want
        th.join()
        g.close()
        g = res["g"]
    assert g.count(stream=sc) == want
    g.close()
