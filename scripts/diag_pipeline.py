"""Pipelined e2e timeline (C3): per step, how long the main thread waits for graph i+1's
build (second host thread, own stream) and how long graph i's count and close take."""
import sys, time, os, concurrent.futures
sys.path.insert(0, os.getcwd())
import numpy as np, torch, tcgen
import paper_conf_ipps_li0ptz24_b200 as tc
src, dst, n = tcgen.CONFIGS["C3"].generate(1)
ps = torch.from_numpy(src).pin_memory(); pd = torch.from_numpy(dst).pin_memory()
sb, sc = torch.cuda.Stream(), torch.cuda.Stream()
def build():
    t0 = time.perf_counter()
    with torch.cuda.stream(sb):
        g = tc.build_csr_host(ps, pd, n, stream=sb)
    return g, t0, time.perf_counter()
# serial reference
for i in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    g, _, _ = build(); T = g.count(stream=sc); g.close(); torch.cuda.synchronize()
    print("serial", round((time.perf_counter() - t0) * 1e3, 1), T, flush=True)
with concurrent.futures.ThreadPoolExecutor(1) as pool:
    torch.cuda.synchronize(); w0 = time.perf_counter()
    fut = pool.submit(build)
    for i in range(6):
        a = time.perf_counter(); g, b0, b1 = fut.result(); b = time.perf_counter()
        if i + 1 < 6: fut = pool.submit(build)
        T = g.count(stream=sc); c = time.perf_counter()
        g.close(); d = time.perf_counter()
        print(f"step {i}: wait build {1e3*(b-a):6.1f}  build ran {1e3*(b0-w0):7.1f}..{1e3*(b1-w0):7.1f}  count {1e3*(c-b):6.1f}  close {1e3*(d-c):6.1f}  t={1e3*(d-w0):7.1f}", flush=True)
    torch.cuda.synchronize(); print("pipelined per step", round((time.perf_counter()-w0)*1e3/6, 1))
