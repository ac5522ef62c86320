"""Diagnostic: per-iteration phases of the e2e leg (pinned host pairs -> T) on
one GPU, with a resident graph and the flush buffer alive as in bench.py."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_li0ptz24_b200 as tc  # noqa: E402
import tcgen  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 12
src, dst, n = tcgen.CONFIGS[cfg].generate(1)
ps, pd = torch.from_numpy(src).pin_memory(), torch.from_numpy(dst).pin_memory()
g0 = tc.build_csr(ps.cuda(), pd.cuda(), n)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def ev():
    e = torch.cuda.Event(enable_timing=True)
    e.record()
    return e


for it in range(iters):
    torch.cuda.synchronize()
    tw = time.perf_counter()
    e0 = ev()
    g = tc.build_csr_host(ps, pd, n)
    e1 = ev()
    tb = time.perf_counter()
    b = g.partition(1)
    o = g.count_range(b[0], b[1])
    t = int(o.item())
    e2 = ev()
    torch.cuda.synchronize()
    te = time.perf_counter()
    ms = {k[3:]: round(v, 1) for k, v in g.info.as_dict().items() if k.startswith("ms_")}
    g.close()
    tcl = time.perf_counter()
    print(f"iter {it}: build_host {e0.elapsed_time(e1):.1f} ms (wall {1e3 * (tb - tw):.1f}) "
          f"count {e1.elapsed_time(e2):.1f}  total wall {1e3 * (te - tw):.1f}  close {1e3 * (tcl - te):.1f}  "
          f"phases {ms}", flush=True)
