"""Diagnostic: time the pieces of the e2e path (host edges -> T) on one GPU."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, numpy as np
import tcgen
import paper_conf_ipps_li0ptz24_b200 as tc

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
t0 = time.time(); src, dst, n = tcgen.CONFIGS[cfg].generate(1); print(f"gen {time.time()-t0:.1f}s pairs {len(src)}", flush=True)
ps, pd = torch.from_numpy(src).pin_memory(), torch.from_numpy(dst).pin_memory()
def ev():
    e = torch.cuda.Event(enable_timing=True); e.record(); return e
for it in range(3):
    torch.cuda.synchronize()
    e0 = ev()
    ds, dd = ps.cuda(non_blocking=True), pd.cuda(non_blocking=True)
    e1 = ev()
    g = tc.build_csr(ds, dd, n)
    e2 = ev()
    t = g.count()
    e3 = ev()
    torch.cuda.synchronize()
    print(f"iter {it}: h2d {e0.elapsed_time(e1):.1f} ms  build {e1.elapsed_time(e2):.1f} ms  count {e2.elapsed_time(e3):.1f} ms  T={t}  info={ {k: round(v,1) if isinstance(v,float) else v for k,v in g.info.as_dict().items() if k.startswith('ms_') or k in ('m','n','m_live','n_chunks','smem_bytes')} }", flush=True)
    g.close(); del ds, dd
for it in range(2):
    torch.cuda.synchronize(); e0 = ev()
    g = tc.build_csr_host(ps, pd, n)
    e1 = ev(); t = g.count(); e2 = ev(); torch.cuda.synchronize()
    print(f"host-entry iter {it}: build_host {e0.elapsed_time(e1):.1f} ms count {e1.elapsed_time(e2):.1f} ms", flush=True)
    g.close()
print("mem peak GB", torch.cuda.max_memory_allocated()/1e9, "free/total", [x/1e9 for x in torch.cuda.mem_get_info()])
# bench-like: a resident graph + flush buffer alive while the host entry runs
g0 = tc.build_csr(ps.cuda(), pd.cuda(), n)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for it in range(3):
    torch.cuda.synchronize(); e0 = ev(); tw = time.perf_counter()
    g = tc.build_csr_host(ps, pd, n)
    e1 = ev(); tb = time.perf_counter()
    b = g.partition(1); o = g.count_range(b[0], b[1]); t = int(o.item())
    info_ms = {k: v for k, v in g.info.as_dict().items() if k.startswith("ms_")}
    e2 = ev(); torch.cuda.synchronize(); te = time.perf_counter()
    g.close(); tc_ = time.perf_counter()
    print(f"resident-graph iter {it}: build_host {e0.elapsed_time(e1):.1f} ms (wall {1e3*(tb-tw):.1f}) count+item {e1.elapsed_time(e2):.1f} ms  total wall {1e3*(te-tw):.1f}  close {1e3*(tc_-te):.1f}", flush=True)
    print("   phases", {k: round(v, 1) for k, v in info_ms.items()}, flush=True)
