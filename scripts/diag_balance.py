"""Per-range timing of tc_partition's split, emulated on one GPU.

    python scripts/diag_balance.py [--config C3] [--worlds 2,4,8] [--reps 3]

Builds the config's graph once, then for every world size P times each rank's
tc_count_range with CUDA events (L2 flushed by a 512 MiB write before every
range, median of --reps) and prints one JSON line per P: per-range ms,
max/mean, and the partials' sum against T.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_li0ptz24_b200 as tc  # noqa: E402
import tcgen  # noqa: E402


def time_range(g, b, e, flush, reps, out):
    ts = []
    s = torch.cuda.current_stream()
    for i in range(reps):
        flush.fill_(i & 0xFF)
        x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        x0.record(s)
        g.count_range(b, e, out=out)
        x1.record(s)
        torch.cuda.synchronize()
        ts.append(x0.elapsed_time(x1))
    return statistics.median(ts), int(out.item()) & (2**64 - 1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--worlds", default="2,4,8")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--calibrate", action="store_true")
    a = ap.parse_args()
    tcgen.lib().tcgen_set_threads(0)
    src, dst, n = tcgen.CONFIGS[a.config].generate(1)
    g = tc.build_csr(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), n)
    del src, dst
    out = torch.zeros(1, dtype=torch.int64, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    T = g.count()
    w = None
    if a.calibrate:
        w = g.calibrate()
        print(json.dumps({"profile_ms": w.round(3).tolist()}), flush=True)
    full, _ = time_range(g, 0, g.m_live, flush, a.reps, out)
    for P in [int(x) for x in a.worlds.split(",")]:
        b = g.partition(P, w) if w is not None else g.partition(P)
        ms, parts = [], []
        for r in range(P):
            t, p = time_range(g, b[r], b[r + 1], flush, a.reps, out)
            ms.append(t)
            parts.append(p)
        mean = sum(ms) / P
        print(json.dumps({"config": a.config, "P": P, "full_ms": full, "range_ms": ms,
                          "max_over_mean": max(ms) / mean, "sum_ms": sum(ms),
                          "bounds": b, "sum_ok": (sum(parts) & (2**64 - 1)) == T}), flush=True)
    g.close()


if __name__ == "__main__":
    main()
