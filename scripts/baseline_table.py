"""BASELINE.md §3 table from one evidence run's committed files (profiles/TAG_*).

usage: python scripts/baseline_table.py TAG   (prints markdown)
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = os.path.join(ROOT, "profiles")


def load(name):
    p = os.path.join(P, name)
    return json.load(open(p)) if os.path.exists(p) else None


def main():
    tag = sys.argv[1]
    ora = {}
    p = os.path.join(P, f"{tag}_oracle_times.jsonl")
    if os.path.exists(p):
        for line in open(p):
            d = json.loads(line)
            ora.setdefault(d["config"], {})[d["threads"]] = d
    ncu = load("ncu_summary.json") or {}
    rows = []
    for cfg in ("C1", "C2", "C3", "C4", "C5"):
        b = load(f"{tag}_bench_{cfg.lower()}.json")
        if not b:
            continue
        r = b["roofline"]
        o = ora.get(cfg, {})
        o1 = o.get(1)
        oall = max(o.values(), key=lambda d: d["threads"]) if o else None
        ot = (f"{oall['threads']}" + (" / 1" if o1 else "")) if oall else "—"
        ob = (f"{oall['build_ms']:.0f}" + (f" / {o1['build_ms']:.0f}" if o1 else "")) if oall else "—"
        oc = (f"{oall['count_ms']:.1f}" + (f" / {o1['count_ms']:.1f}" if o1 else "")) if oall else "—"
        nk = (ncu.get(cfg) or {}).get("kernels", {})
        kn = "k_count" if r["kernel"].startswith("k_count (") else "k_count_flat"
        k = nk.get(kn) if (ncu.get(cfg) or {}).get("tag") == tag else None
        dram = f"{k['dram_gbs']:.0f}" if k and "dram_gbs" in k else "—"
        l2 = f"{k['lts_gbs']:.0f}" if k and "lts_gbs" in k else "—"
        e2e = b.get("e2e") or {}
        rows.append(f"| {cfg} | {ot} | {ob} | {oc} | {b['build_ms']['total_events']:.1f} | "
                     f"{b['ms_per_step']:.3f} | {b['value'] / 1e9:.2f} G | "
                     f"{r['frac']:.2f} ({kn}) / {r['step']['frac']:.2f} | {dram} | {l2} | "
                     f"{e2e.get('ms_per_step', float('nan')):.1f} |")
    print("| Config | Oracle threads (all / 1) | Oracle build ms | Oracle count ms | GPU build ms | "
          "GPU count ms | oriented edges/s | method-bytes roofline frac (dominant kernel / step) | "
          "ncu DRAM GB/s | ncu L2 GB/s | e2e ms |")
    print("|---|---|---|---|---|---|---|---|---|---|---|")
    print("\n".join(rows))


if __name__ == "__main__":
    main()
