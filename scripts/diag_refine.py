"""Balance of the measured-profile split vs slices K and one refinement pass.

    python scripts/diag_refine.py --config C4 --P 8 --slices 64,128,256

For each K: calibrate, split, time every range alone (L2 flushed, median of 3),
then REFINE once: scale every slice's ms by (measured / predicted time) of the
range holding it, split again and time again.  One JSON line per K.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_li0ptz24_b200 as tc  # noqa: E402
import tcgen  # noqa: E402


def time_ranges(g, b, flush, out, reps=3):
    s = torch.cuda.current_stream()
    res = []
    for r in range(len(b) - 1):
        ts = []
        for i in range(reps):
            flush.fill_(i)
            x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            x0.record(s)
            g.count_range(b[r], b[r + 1], out=out)
            x1.record(s)
            torch.cuda.synchronize()
            ts.append(x0.elapsed_time(x1))
        res.append(statistics.median(ts))
    return res


def predicted(seg, cost, first, w, b):
    """Profile time of each range [b_r, b_r+1) (chunk-aligned)."""
    W = np.zeros(len(cost))
    acc = 0.0
    for i in range(len(w)):
        c0, c1 = first[i], first[i + 1]
        span = cost[c1] - cost[c0]
        if c1 > c0:
            W[c0:c1] = acc + (w[i] * (cost[c0:c1] - cost[c0]) / span if span > 0 else 0.0)
        acc += w[i]
    W[-1] = acc
    idx = [int(np.searchsorted(seg, x)) for x in b]
    return [W[idx[r + 1]] - W[idx[r]] for r in range(len(b) - 1)], idx


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--P", type=int, default=8)
    ap.add_argument("--slices", default="64,128,256")
    a = ap.parse_args()
    tcgen.lib().tcgen_set_threads(0)
    src, dst, n = tcgen.CONFIGS[a.config].generate(1)
    g = tc.build_csr(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), n)
    del src, dst
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    out = torch.zeros(1, dtype=torch.int64, device="cuda")
    seg, cost = g.chunks()
    nl = int(g.info.n_long_chunks)
    for K in [int(x) for x in a.slices.split(",")]:
        w = g.calibrate(K)
        first = tc.slice_bounds(cost, nl, K)
        b = g.partition(a.P, w)
        t = time_ranges(g, b, flush, out)
        p, idx = predicted(seg, cost, first, w, b)
        f = [ti / pi for ti, pi in zip(t, p)]
        # refine: slice i scaled by the factor of the range holding its midpoint chunk
        w2 = w.copy()
        for i in range(K):
            mid = (first[i] + first[i + 1]) // 2
            r = max(0, min(a.P - 1, int(np.searchsorted(idx, mid, side="right")) - 1))
            w2[i] = w[i] * f[r]
        b2 = g.partition(a.P, w2)
        t2 = time_ranges(g, b2, flush, out)
        mm = lambda x: max(x) / (sum(x) / len(x))
        print(json.dumps({"config": a.config, "P": a.P, "K": K, "max_over_mean": mm(t),
                          "range_ms": [round(x, 2) for x in t], "pred_factor": [round(x, 3) for x in f],
                          "refined_max_over_mean": mm(t2), "refined_range_ms": [round(x, 2) for x in t2]}),
              flush=True)


if __name__ == "__main__":
    main()
