"""Copy one gpu_evidence.sh run (gpurun_out/TAG_*) into profiles/ and summarise it.

usage: python scripts/collect_evidence.py TAG

  profiles/TAG_bench_*.json, TAG_reference_c3.json       the JSON lines as printed
  profiles/TAG_pytest_gpu.txt, TAG_smoke.txt              test / smoke logs
  profiles/TAG_sanitize_{racecheck,synccheck,memcheck}.txt
  profiles/TAG_oracle_times.jsonl                          oracle build/count ms (1 / all threads)
  profiles/TAG_c3_launches.txt                             per-kernel share of the ncu launch list
  profiles/TAG_{c3,c2}_ncu.txt + profiles/ncu_summary.json (scripts/profile_summary.py)
"""
import csv
import glob
import json
import os
import shutil
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
O = os.path.join(ROOT, "gpurun_out")
P = os.path.join(ROOT, "profiles")


def launches(tag):
    p = os.path.join(O, f"{tag}_launches_c3.csv")
    if not os.path.exists(p):
        return
    rows = [r for r in csv.reader(open(p)) if len(r) > 10]
    hdr = rows[0]
    ki, mi, vi, ui = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    tot, cnt = defaultdict(float), defaultdict(int)
    for r in rows[1:]:
        if r[mi] != "gpu__time_duration.sum":
            continue
        v = float(r[vi].replace(",", ""))
        v *= {"ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0}.get(r[ui], 1.0)
        name = r[ki].split("(")[0]
        tot[name] += v
        cnt[name] += 1
    s = sum(tot.values())
    with open(os.path.join(P, f"{tag}_c3_launches.txt"), "w") as f:
        f.write(f"# {tag}: ncu --metrics gpu__time_duration.sum --clock-control none launch list of\n"
                "# `python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded "
                "--no-balance` (C3: two builds + 3 count steps; cold-cache, serialised: compare "
                "shares, not absolutes)\n")
        f.write(f"{'total ms':>10} {'launches':>8} {'share':>6}  kernel\n")
        for k, v in sorted(tot.items(), key=lambda x: -x[1]):
            f.write(f"{v:10.3f} {cnt[k]:8d} {100 * v / s:5.1f}%  {k[:150]}\n")


def main():
    tag = sys.argv[1]
    os.makedirs(P, exist_ok=True)
    for pat in ("bench_*.json", "reference_c3.json", "pytest_gpu.txt", "smoke.txt", "sanitize_*.txt",
                "oracle_times.jsonl"):
        for f in glob.glob(os.path.join(O, f"{tag}_{pat}")):
            shutil.copy(f, P)
    launches(tag)
    h = open(os.path.join(O, f"{tag}_src_hash.txt")).read().strip()
    for cfg in ("C3", "C2"):
        rep = os.path.join(O, f"{tag}_{cfg.lower()}_count.ncu-rep")
        if os.path.exists(rep):
            subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "profile_summary.py"), rep, tag,
                            cfg, "--src-hash", h], check=True, stdout=subprocess.DEVNULL)
    print("collected", tag, "src_hash", h)


if __name__ == "__main__":
    main()
