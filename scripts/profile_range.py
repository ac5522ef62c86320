"""Count one slice of the plan (for ncu): the live edges of chunks covering
cost fraction [--lo, --hi) of the long class (or --short: of the short class).

    ncu ... python scripts/profile_range.py --config C3 --lo 0 --hi 0.05
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_li0ptz24_b200 as tc  # noqa: E402
import tcgen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--lo", type=float, default=0.0)
ap.add_argument("--hi", type=float, default=0.05)
ap.add_argument("--short", action="store_true")
ap.add_argument("--opt", action="append", default=[])
a = ap.parse_args()
src, dst, n = tcgen.CONFIGS[a.config].generate(1)
opts = {k: int(v) for k, v in (kv.split("=") for kv in a.opt)} or None
g = tc.build_csr(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), n, options=opts)
seg, cost = g.chunks()
nl = int(g.info.n_long_chunks)
c0, c1 = (nl, len(cost) - 1) if a.short else (0, nl)
base, span = cost[c0], cost[c1] - cost[c0]
i0 = int(np.searchsorted(cost[c0:c1 + 1], base + a.lo * span)) + c0
i1 = int(np.searchsorted(cost[c0:c1 + 1], base + a.hi * span)) + c0
out = g.count_range(int(seg[i0]), int(seg[i1]))
out = g.count_range(int(seg[i0]), int(seg[i1]))  # the profiled launch
torch.cuda.synchronize()
info = g.info
print(f"chunks [{i0}, {i1}) edges [{seg[i0]}, {seg[i1]}) partial {int(out.item())}")
