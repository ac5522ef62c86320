"""Oracle (CPU) build and count times on this host, for BASELINE.md §3:
1 thread and all hardware threads on C1, C2, C5; all threads on C3.
One JSON line per (config, threads)."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import tcgen  # noqa: E402

model = "unknown"
for line in open("/proc/cpuinfo"):
    if line.startswith("model name"):
        model = line.split(":", 1)[1].strip()
        break
tcgen.lib().tcgen_set_threads(0)
for cfg, threads in (("C1", 1), ("C1", 0), ("C2", 1), ("C2", 0), ("C5", 1), ("C5", 0), ("C3", 0)):
    src, dst, n = tcgen.CONFIGS[cfg].generate(1)
    t0 = time.perf_counter()
    r = oracle.count(src, dst, n, threads=threads)
    wall = time.perf_counter() - t0
    print(json.dumps({"config": cfg, "threads": r.threads, "triangles": r.triangles, "m": r.m,
                      "build_ms": round(r.build_ms, 2), "count_ms": round(r.count_ms, 2),
                      "wall_s": round(wall, 2), "cpu": model, "nproc": os.cpu_count()}), flush=True)
