"""Where does a slow e2e step (tc_build_csr_host + count + close) spend its time?
Per step: host wall of build / count / close and the build's own phase ms (events)."""
import sys, os, time, gc
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, tcgen
import paper_conf_ipps_li0ptz24_b200 as tc
cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 40
src, dst, n = tcgen.CONFIGS[cfg].generate(1)
ps = torch.from_numpy(src).pin_memory(); pd = torch.from_numpy(dst).pin_memory()
for i in range(steps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    g = tc.build_csr_host(ps, pd, n)
    t1 = time.perf_counter()
    T = g.count()
    t2 = time.perf_counter()
    inf = g.info
    ph = (inf.ms_canon, inf.ms_sort_unique, inf.ms_degree_rank, inf.ms_orient_csr, inf.ms_plan, inf.ms_total)
    g.close()
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    print(f"{i:2d} total {1e3*(t3-t0):7.1f}  build {1e3*(t1-t0):7.1f} (events: " + " ".join(f"{x:6.1f}" for x in ph) +
          f")  count {1e3*(t2-t1):6.1f}  close {1e3*(t3-t2):6.1f}  gc {gc.get_count()}", flush=True)
