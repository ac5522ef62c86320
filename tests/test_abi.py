"""CPU-side checks of the C-ABI boundary (-m "not gpu").

No compute call is made here (there is no GPU in the build container): the
library must load, export every symbol include/tc.h declares, reject bad
arguments before touching the device, and its host-only partition logic must
cut cost prefixes into balanced contiguous ranges.
"""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def tc():
    subprocess.run(["make", "-s", "-C", ROOT, "paper_conf_ipps_li0ptz24_b200/libtc.so"],
                   check=True)
    import paper_conf_ipps_li0ptz24_b200 as tc
    tc.lib()
    return tc


def header_symbols():
    text = open(os.path.join(ROOT, "include", "tc.h")).read()
    return sorted(set(re.findall(r"TC_API\s+[\w\s\*]+?\b(tc_\w+)\s*\(", text)))


def test_header_symbols_match_binding(tc):
    assert header_symbols() == sorted(tc.EXPORTS)


def test_library_exports_every_symbol(tc):
    out = subprocess.run(["nm", "-D", "--defined-only", tc.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (tc_\w+)", out))
    missing = set(header_symbols()) - exported
    assert not missing, missing
    # nothing else leaks from the C-ABI namespace
    assert exported == set(header_symbols())


def test_library_is_sm100a(tc):
    out = subprocess.run(["cuobjdump", "--list-elf", tc.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    assert "sm_100a" in out


def test_version(tc):
    assert tc.version().startswith("b200tc")


def test_null_out_is_invalid(tc):
    L = tc.lib()
    assert L.tc_build_csr(None, None, 0, -1, 0, None, None, None) == tc.TC_ERR_INVALID_ARGUMENT
    assert "out" in L.tc_last_error().decode()


def test_bad_arguments_rejected_before_device(tc):
    L = tc.lib()
    h = ctypes.c_void_p(0)
    assert L.tc_build_csr(None, None, -1, -1, 0, None, None, ctypes.byref(h)) == 1
    assert L.tc_build_csr(None, None, 5, -1, 0, None, None, ctypes.byref(h)) == 1
    assert L.tc_build_csr(None, None, 0, 2**31, 0, None, None, ctypes.byref(h)) == 1
    assert L.tc_build_csr(None, None, 0, -1, 0x80, None, None, ctypes.byref(h)) == 1
    assert h.value is None
    bad = tc.Options(chunk_cost=8)
    assert L.tc_build_csr(None, None, 0, -1, 0, ctypes.byref(bad), None, ctypes.byref(h)) == 1
    bad = tc.Options(block_threads=2048)
    assert L.tc_build_csr(None, None, 0, -1, 0, ctypes.byref(bad), None, ctypes.byref(h)) == 1
    assert L.tc_count(None, None, None) == 1
    assert L.tc_count_range(None, 0, 0, None, None) == 1
    assert L.tc_partition(None, 2, None) == 1
    assert L.tc_partition_measured(None, 2, 1, None, None) == 1
    assert L.tc_plan_chunks(None, None, None) == 1
    assert L.tc_calibrate(None, None, 4, None) == 1
    assert L.tc_slice_bounds(None, 0, 0, 1, None) == 1
    assert L.tc_refine_profile(None, None, 2, 1, None) == 1
    assert L.tc_count_range_fused(None, 0, 0, None, None, None, 1, 1, None, None) == 1
    assert L.tc_graph_info(None, None) == 1
    assert L.tc_support(None, None, None) == 1
    assert L.tc_edge_list(None, None, None, None) == 1
    L.tc_free(None)  # no-op


def test_allocator_hooks_must_pair(tc):
    L = tc.lib()
    cb = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
    f = cb(lambda n, s, c: None)
    assert L.tc_set_allocator(ctypes.cast(f, ctypes.c_void_p), None, None) == 1
    assert L.tc_set_allocator(None, None, None) == 0


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_partition_prefix_balanced(tc, world):
    rng = np.random.default_rng(world)
    cost = rng.integers(1, 200, size=5000)
    prefix = np.concatenate([[0], np.cumsum(cost)])
    b = tc.partition_prefix(prefix, world)
    assert b[0] == 0 and b[-1] == len(cost) and all(x <= y for x, y in zip(b, b[1:]))
    loads = [prefix[b[r + 1]] - prefix[b[r]] for r in range(world)]
    assert sum(loads) == prefix[-1]
    # every part within one unit's cost of the ideal share
    assert max(loads) - prefix[-1] / world <= cost.max()


def test_partition_prefix_degenerate(tc):
    assert tc.partition_prefix([0], 4) == [0, 0, 0, 0, 0]
    assert tc.partition_prefix([0, 10], 3) == [0, 1, 1, 1] or tc.partition_prefix([0, 10], 3)[-1] == 1
    with pytest.raises(tc.InvalidArgument):
        tc.partition_prefix([0, 1], 0)


def test_struct_layouts_match_header(tc, tmp_path):
    """The ctypes mirrors of tc_options / tc_graph_info_t match the C header."""
    src = tmp_path / "sz.c"
    src.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "tc.h"\n'
                   'int main(void){printf("%zu %zu %zu %zu %zu %zu\\n", sizeof(tc_options), '
                   'sizeof(tc_graph_info_t), offsetof(tc_graph_info_t, row_ptr), '
                   'offsetof(tc_graph_info_t, n_long_chunks), '
                   'offsetof(tc_graph_info_t, method_bytes), '
                   'offsetof(tc_graph_info_t, keys_long));return 0;}\n')
    exe = tmp_path / "sz"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    got = [int(x) for x in subprocess.run([str(exe)], capture_output=True, text=True,
                                          check=True).stdout.split()]
    want = [ctypes.sizeof(tc.Options), ctypes.sizeof(tc.GraphInfo), tc.GraphInfo.row_ptr.offset,
            tc.GraphInfo.n_long_chunks.offset, tc.GraphInfo.method_bytes.offset,
            tc.GraphInfo.keys_long.offset]
    assert got == want


def _profile_W(seg, cost, nL, first, ms):
    """The profile's time at every chunk boundary (tc_partition_chunks' W)."""
    W = np.zeros(len(cost))
    acc = 0.0
    for i in range(len(ms)):
        c0, c1 = first[i], first[i + 1]
        span = cost[c1] - cost[c0]
        for c in range(c0, c1):
            W[c] = acc + (ms[i] * (cost[c] - cost[c0]) / span if span > 0 else 0.0)
        acc += ms[i]
    W[-1] = acc
    return W


@pytest.mark.parametrize("K", [1, 2, 7, 64])
def test_slice_bounds(tc, K):
    """Slices cover the chunks in order, never straddle the class boundary and
    split each class at near-equal cost."""
    rng = np.random.default_rng(K)
    nc, nL = 3000, 1800
    cost = np.concatenate([[0], np.cumsum(rng.integers(1, 400, size=nc))])
    f = tc.slice_bounds(cost, nL, K)
    assert f[0] == 0 and f[-1] == nc and all(a <= b for a, b in zip(f, f[1:]))
    if K >= 2:
        assert nL in f  # the class boundary is a slice boundary
    step = np.diff(cost).max()
    for cls0, cls1 in ((0, nL), (nL, nc)):
        inner = [i for i in range(K) if cls0 <= f[i] and f[i + 1] <= cls1 and f[i + 1] > f[i]]
        if len(inner) > 1:
            sizes = [cost[f[i + 1]] - cost[f[i]] for i in inner]
            assert max(sizes) - min(sizes) <= 2 * step
    assert tc.slice_bounds(cost, 0, 4)[-1] == nc and tc.slice_bounds(cost, nc, 4)[-1] == nc


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("K", [2, 16, 64])
def test_partition_chunks_profile_balance(tc, world, K):
    """cuts on the profile-weighted cost prefix; every range
    within one chunk's weight of the ideal share, chunk-aligned, covering
    [0, m_live); a non-uniform profile moves the cuts."""
    rng = np.random.default_rng(world * 100 + K)
    nc, nL = 3000, 1800
    cost = np.concatenate([[0], np.cumsum(rng.integers(1, 400, size=nc))])
    seg = np.concatenate([[0], np.cumsum(rng.integers(1, 50, size=nc))])
    ms = rng.uniform(0.5, 3.0, size=K)
    b = tc.partition_chunks(seg, cost, nL, ms, world)
    assert b[0] == 0 and b[-1] == seg[-1] and all(x <= y for x, y in zip(b, b[1:]))
    assert set(b) <= set(seg.tolist())
    W = _profile_W(seg, cost, nL, tc.slice_bounds(cost, nL, K), ms)
    assert abs(W[-1] - ms.sum()) < 1e-9 * ms.sum()
    idx = [int(np.searchsorted(seg, x)) for x in b]
    loads = [W[idx[r + 1]] - W[idx[r]] for r in range(world)]
    assert max(abs(x - W[-1] / world) for x in loads) <= np.diff(W).max() + 1e-12


def test_partition_chunks_profile_moves_the_cut(tc):
    """A slower long class pulls the 2-way cut toward the front."""
    seg = np.arange(11, dtype=np.int64) * 10
    cost = np.arange(11, dtype=np.int64) * 100  # 10 equal chunks, 5 long
    assert tc.slice_bounds(cost, 5, 2) == [0, 5, 10]
    assert tc.partition_chunks(seg, cost, 5, [1.0, 1.0], 2) == [0, 50, 100]
    assert tc.partition_chunks(seg, cost, 5, [1.0, 3.0], 2)[1] == 70  # W: 1 + 3 -> cut at 2
    assert tc.partition_chunks(seg, cost, 5, [3.0, 1.0], 2)[1] == 30
    with pytest.raises(tc.InvalidArgument):
        tc.partition_chunks(seg, cost, 5, [-1.0, 1.0], 2)
    with pytest.raises(tc.InvalidArgument):
        tc.partition_chunks(seg[::-1].copy(), cost, 5, [1.0, 1.0], 2)
