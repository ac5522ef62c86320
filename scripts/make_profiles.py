"""Turn a gpurun capture into the committed evidence under profiles/.

usage: python scripts/make_profiles.py TAG [CONFIG]
  reads  gpurun_out/TAG_prof_c3.ncu-rep  (ncu --set full of one k_count launch)
         gpurun_out/TAG_launches_c3.csv  (ncu --metrics gpu__time_duration.sum launch list)
  writes profiles/TAG_<cfg>_count_ncu.txt   headline counters + stalls + hottest SASS
         profiles/TAG_<cfg>_launches.txt    per-kernel share of the launch list
         profiles/ncu_summary.json          {cfg: {...}} read by bench.py for roofline.traffic
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "profiles")


def raw_metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (vals[i], units[i]) for i, h in enumerate(hdr)}


def to_bytes(v, unit):
    x = float(v.replace(",", ""))
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def to_ms(v, unit):
    x = float(v.replace(",", ""))
    return x * {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1, "msecond": 1, "s": 1e3}.get(unit, 1)


def main():
    tag = sys.argv[1]
    cfg = sys.argv[2] if len(sys.argv) > 2 else "C3"
    low = cfg.lower()
    os.makedirs(OUT, exist_ok=True)
    rep = os.path.join(ROOT, "gpurun_out", f"{tag}_prof_{low}.ncu-rep")
    summary = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "ncu_summary.py"), rep,
                              "--sass", "40"], capture_output=True, text=True, check=True).stdout
    with open(os.path.join(OUT, f"{tag}_{low}_count_ncu.txt"), "w") as f:
        f.write(f"# ncu --set full --clock-control none, one k_count launch, config {cfg} ({tag})\n")
        f.write(summary)
    m = raw_metrics(rep)
    dram = to_bytes(*m["dram__bytes_read.sum"]) + to_bytes(*m["dram__bytes_write.sum"])
    ms = to_ms(*m["gpu__time_duration.sum"])
    # the short-class kernel of the same count step, if captured
    rep_flat = os.path.join(ROOT, "gpurun_out", f"{tag}_prof_{low}_flat.ncu-rep")
    flat = None
    if os.path.exists(rep_flat):
        mf = raw_metrics(rep_flat)
        flat = {"dram_bytes": to_bytes(*mf["dram__bytes_read.sum"]) + to_bytes(*mf["dram__bytes_write.sum"]),
                "ms": to_ms(*mf["gpu__time_duration.sum"])}
        summary_flat = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "ncu_summary.py"),
                                       rep_flat], capture_output=True, text=True, check=True).stdout
        with open(os.path.join(OUT, f"{tag}_{low}_count_flat_ncu.txt"), "w") as f:
            f.write(f"# ncu --set full --clock-control none, one k_count_flat launch, config {cfg} ({tag})\n")
            f.write(summary_flat)
    entry = {"round_tag": tag,
             "dram_bytes_per_launch": dram + (flat["dram_bytes"] if flat else 0.0),
             "what": "k_count (long class) + k_count_flat (short class) of one count step",
             "k_count_dram_bytes": dram, "k_count_flat": flat, "kernel_ms_under_ncu": ms,
             "dram_gbs": dram / ms / 1e6, "lts_bytes": to_bytes(*m["lts__t_bytes.sum"]) if "lts__t_bytes.sum" in m else None,
             "issue_active_pct": float(m["smsp__issue_active.avg.pct_of_peak_sustained_active"][0]),
             "warps_active_pct": float(m["sm__warps_active.avg.pct_of_peak_sustained_active"][0]),
             "l2_hit_pct": float(m["lts__t_sector_hit_rate.pct"][0]),
             "warp_efficiency": float(m["smsp__thread_inst_executed_per_inst_executed.ratio"][0]) / 32,
             "sm_cycles_active_min_avg_max": [float(m[f"sm__cycles_active.{k}"][0].replace(",", ""))
                                              for k in ("min", "avg", "max")]}
    lpath = os.path.join(ROOT, "gpurun_out", f"{tag}_launches_{low}.csv")
    if os.path.exists(lpath):
        rows = list(csv.DictReader(l for l in open(lpath) if not l.startswith("==")))
        agg = defaultdict(lambda: [0, 0.0])
        for r in rows:
            if r["Metric Name"] != "gpu__time_duration.sum":
                continue
            k = r["Kernel Name"].split("(")[0]
            agg[k][0] += 1
            agg[k][1] += to_ms(r["Metric Value"], r["Metric Unit"])
        tot = sum(v[1] for v in agg.values())
        with open(os.path.join(OUT, f"{tag}_{low}_launches.txt"), "w") as f:
            f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none launch list of\n"
                    f"# `python bench.py --config {cfg} --steps 2 --warmup 1 --no-e2e --no-cpu-baseline`\n"
                    f"# (two builds + 3 counts; cold-cache, serialised: compare shares, not absolutes)\n")
            f.write(f"{'total ms':>10} {'launches':>8} {'share':>6}  kernel\n")
            for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
                f.write(f"{v[1]:10.3f} {v[0]:8d} {100 * v[1] / tot:5.1f}%  {k}\n")
        cnt = agg.get("tc::<unnamed>::k_count", [0, 0])
        entry["launch_list_k_count_ms_per_launch"] = cnt[1] / max(1, cnt[0])
        entry["launch_list_k_count_share"] = cnt[1] / tot if tot else None
    p = os.path.join(OUT, "ncu_summary.json")
    data = json.load(open(p)) if os.path.exists(p) else {}
    data[cfg] = entry
    json.dump(data, open(p, "w"), indent=1, sort_keys=True)
    print(json.dumps(entry, indent=1))


if __name__ == "__main__":
    main()
