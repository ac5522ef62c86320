"""Measured balance of the multi-GPU edge ranges, emulated
on one B200: every rank's tc_count_range of the tc_partition_measured split
(profile = this device's tc_calibrate, 64 slices, refined for P ranks by
tc_refine_profile, as agreed_profile does) is timed alone with CUDA
events, L2 flushed before each (median of 5); the slowest range may exceed the mean by at
most 5 %, and the partials sum to the oracle's stored T (the per-edge
intersections are independent, so any cut is exact)."""
import json
import os
import statistics

import numpy as np
import pytest

import tcgen

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

BALANCE_MAX = 1.05


@pytest.fixture(scope="module")
def tc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_li0ptz24_b200 as tc
    tc.lib()
    return tc


def _range_ms(g, b, e, flush, out, reps=5):
    s = torch.cuda.current_stream()
    ts = []
    for i in range(reps):
        flush.fill_(i)
        x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        x0.record(s)
        g.count_range(b, e, out=out)
        x1.record(s)
        torch.cuda.synchronize()
        ts.append(x0.elapsed_time(x1))
    return statistics.median(ts), int(out.item()) & (2**64 - 1)


@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_partition_balance_measured(tc, cfg):
    stored = json.load(open(os.path.join(os.path.dirname(__file__), "golden",
                                         "config_counts.json")))[f"{cfg}/seed1"]
    src, dst, n = tcgen.CONFIGS[cfg].generate(1)
    ds, dd = torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda()
    del src, dst
    with tc.build_csr(ds, dd, n) as g:
        del ds, dd
        w = g.calibrate()
        assert (w >= 0).all() and w.sum() > 0
        flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
        out = torch.zeros(1, dtype=torch.int64, device="cuda")
        report = {}
        for P in (2, 4, 8):
            b = g.partition(P, g.refine(P, w))
            res = [_range_ms(g, b[r], b[r + 1], flush, out) for r in range(P)]
            ms = [t for t, _ in res]
            assert sum(p for _, p in res) & (2**64 - 1) == stored["triangles"]
            report[P] = (max(ms) / (sum(ms) / P), [round(t, 3) for t in ms])
        del flush
        print(cfg, "profile ms", np.round(w, 3).tolist(), report)
        for P, (ratio, ms) in report.items():
            assert ratio <= BALANCE_MAX, f"{cfg} P={P}: max/mean {ratio:.3f} {ms}"
