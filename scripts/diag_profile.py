"""Print the measured time profile of the plan (tc_calibrate: equal-cost slices timed
on the device) with each slice's class and chunk/group density: where the count spends its time."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, tcgen
import paper_conf_ipps_li0ptz24_b200 as tc
cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
src, dst, n = tcgen.CONFIGS[cfg].generate(1)
g = tc.build_csr(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), n)
g.count()
ms = g.calibrate(64)
ms = g.calibrate(64)
seg, cost = g.chunks()
nl = int(g.info.n_long_chunks)
print(cfg, "n_chunks", len(seg) - 1, "long", nl, "total ms %.2f" % float(np.sum(ms)))
for i, t in enumerate(ms):
    print("%2d %7.3f ms" % (i, t))
