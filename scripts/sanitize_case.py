"""Small counts for compute-sanitizer (racecheck / synccheck / memcheck):
C1 and RMAT-12 through both count kernels (long_min=32 puts the long class on
the warp-specialised k_count with its mbarrier slot ring), the support kernel,
and the fused epilogue; every result checked against the oracle."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_li0ptz24_b200 as tc  # noqa: E402
import tcgen  # noqa: E402


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


cases = [tcgen.CONFIGS["C1"].generate(1), tcgen.rmat(12, 16, 4)]
for src, dst, n in cases:
    want = oracle.triangles(src, dst, n)
    for opts in ({"long_min": 32}, {"long_min": 32, "bitmap_factor": -1}, None):
        with tc.build_csr(dev(src), dev(dst), n, options=opts) as g:
            assert g.count() == want, (g.count(), want)
            sup = g.support()
            assert int(sup.to(torch.int64).sum().item()) == 3 * want
    with tc.build_csr(dev(src), dev(dst), n, options={"long_min": 32}) as g:
        fs = tc.FusedSum(mode="peers")
        assert tc.count_partitioned(g, fused=fs) == want
        fs.close()
print("sanitize cases OK")
