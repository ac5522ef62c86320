import sys, os, statistics, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch, tcgen
import paper_conf_ipps_li0ptz24_b200 as tc
cfg = sys.argv[1]
src, dst, n = tcgen.CONFIGS[cfg].generate(1)
ds, dd = torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(); del src, dst
g = tc.build_csr(ds, dd, n); del ds, dd
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda"); out = torch.zeros(1, dtype=torch.int64, device="cuda")
def rms(b, e):
    ts = []
    for i in range(5):
        flush.fill_(i); x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s = torch.cuda.current_stream(); x0.record(s); g.count_range(b, e, out=out); x1.record(s); torch.cuda.synchronize(); ts.append(x0.elapsed_time(x1))
    return statistics.median(ts)
for rep in range(2):
    w = g.calibrate()
    for P in (4, 8):
        r1 = g.refine(P, w); r2 = g.refine(P, r1)
        for name, prof in (("1 pass", r1), ("2 passes", r2)):
            b = g.partition(P, prof); ms = [rms(b[r], b[r+1]) for r in range(P)]
            print(cfg, rep, P, name, round(max(ms)/(sum(ms)/P), 4), [round(x,2) for x in ms], flush=True)
