"""Overlap diagnostics for the pipelined e2e leg (C3): does a pinned H2D copy
overlap a count on another stream, and does a host build?"""
import sys, time, os, threading
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, tcgen
import paper_conf_ipps_li0ptz24_b200 as tc
src, dst, n = tcgen.CONFIGS["C3"].generate(1)
ps = torch.from_numpy(src).pin_memory(); pd = torch.from_numpy(dst).pin_memory()
sb, sc = torch.cuda.Stream(), torch.cuda.Stream()
g = tc.build_csr_host(ps, pd, n)
ds = torch.empty_like(ps, device="cuda"); dd = torch.empty_like(pd, device="cuda")
out = torch.zeros(1, dtype=torch.int64, device="cuda")
def h2d():
    with torch.cuda.stream(sb):
        ds.copy_(ps, non_blocking=True); dd.copy_(pd, non_blocking=True)
def cnt():
    g.count_async(out=out, stream=sc)
def timed(name, *fns):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    for f in fns: f()
    torch.cuda.synchronize(); print(f"{name:40s} {1e3*(time.perf_counter()-t0):8.1f} ms", flush=True)
for _ in range(2):
    timed("h2d alone", h2d); timed("count alone", cnt); timed("h2d + count (both enqueued)", h2d, cnt)
    timed("count + h2d (both enqueued)", cnt, h2d)
# build in a thread while counts run back to back on sc
for _ in range(2):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    res = {}
    def b():
        with torch.cuda.stream(sb):
            res["g"] = tc.build_csr_host(ps, pd, n, stream=sb)
        res["t"] = time.perf_counter() - t0
    th = threading.Thread(target=b); th.start()
    time.sleep(0.002)
    cnt(); torch.cuda.current_stream().synchronize()
    sc.synchronize(); tc_end = time.perf_counter() - t0
    th.join(); res["g"].close()
    print(f"build in thread + 1 count: count done {1e3*tc_end:7.1f} ms, build done {1e3*res['t']:7.1f} ms", flush=True)
torch.cuda.synchronize(); t0 = time.perf_counter()
g2 = tc.build_csr_host(ps, pd, n, stream=sb); print("build alone", round(1e3*(time.perf_counter()-t0),1)); g2.close()
