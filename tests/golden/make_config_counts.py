"""Writes tests/golden/config_counts.json: the CPU oracle's exact triangle
count (and m, n', max d+) for each BASELINE.json config at the seeds the
bench and tests use.  Calls only oracle/ and tcgen/ (never the CUDA path),
so these stored values are oracle values.

    python tests/golden/make_config_counts.py C1 C2 C3 C5 [--seed 1]
"""
import argparse
import json
import os
import sys
import time

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import tcgen  # noqa: E402

PATH = os.path.join(HERE, "config_counts.json")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="+")
    ap.add_argument("--seed", type=int, default=1)
    a = ap.parse_args()
    data = json.load(open(PATH)) if os.path.exists(PATH) else {}
    for c in a.configs:
        t0 = time.time()
        src, dst, n = tcgen.CONFIGS[c].generate(a.seed)
        gen_s = time.time() - t0
        r = oracle.count(src, dst, n)
        data[f"{c}/seed{a.seed}"] = {
            "config": tcgen.CONFIGS[c].description, "seed": a.seed, "pairs": int(len(src)),
            "checksum": tcgen.checksum(src, dst), "n": int(n), "n_active": r.n_active,
            "m": r.m, "max_out_degree": r.max_out_degree, "triangles": r.triangles,
            "oracle_threads": r.threads, "oracle_build_ms": round(r.build_ms, 1),
            "oracle_count_ms": round(r.count_ms, 1), "merge_steps": r.merge_steps_total,
        }
        print(c, data[f"{c}/seed{a.seed}"], f"gen {gen_s:.1f}s", flush=True)
        json.dump(data, open(PATH, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
