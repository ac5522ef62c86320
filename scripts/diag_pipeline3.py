"""Pipelined e2e variants (C3): which part of the loop serialises build i+1 with count i."""
import sys, time, os, concurrent.futures
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, tcgen
import paper_conf_ipps_li0ptz24_b200 as tc
src, dst, n = tcgen.CONFIGS["C3"].generate(1)
ps = torch.from_numpy(src).pin_memory(); pd = torch.from_numpy(dst).pin_memory()
sb, sc = torch.cuda.Stream(), torch.cuda.Stream()
out = torch.zeros(1, dtype=torch.int64, device="cuda")
def build():
    t0 = time.perf_counter()
    with torch.cuda.stream(sb):
        g = tc.build_csr_host(ps, pd, n, stream=sb)
    return g, t0, time.perf_counter()
g, _, _ = build(); g.count(); g.close()
def run(name, count_mode, close_now, k=6):
    keep = []
    with concurrent.futures.ThreadPoolExecutor(1) as pool:
        torch.cuda.synchronize(); w0 = time.perf_counter()
        fut = pool.submit(build)
        for i in range(k):
            g, b0, b1 = fut.result()
            if i + 1 < k: fut = pool.submit(build)
            if count_mode == "sync":
                T = g.count(stream=sc)
            else:
                g.count_async(out=out, stream=sc); sc.synchronize(); T = int(out.item())
            if close_now: g.close()
            else: keep.append(g)
        torch.cuda.synchronize()
        per = (time.perf_counter() - w0) * 1e3 / k
    for x in keep: x.close()
    print(f"{name:44s} per step {per:7.1f} ms (build {1e3*(b1-b0):6.1f} last)", flush=True)
for rep in range(2):
    run("count() + close each step", "sync", True)
    run("count_async(out) + close each step", "async", True)
    run("count() + close at the end", "sync", False)
    run("count_async(out) + close at the end", "async", False)
