"""Turn one ncu --set full capture of a count step into committed evidence.

usage: python scripts/profile_summary.py REP.ncu-rep TAG [CONFIG] [--src-hash H]

REP holds the count kernels of one step (k_count = long class, k_count_flat =
short class; the last launch of each is used).  Writes
  profiles/TAG_<cfg>_ncu.txt      headline counters, stalls, top source lines
  profiles/ncu_summary.json       {cfg: {src_hash, tag, kernels: {name: {...}}}}
bench.py reports roofline.traffic from ncu_summary.json only when its
src_hash equals the hash of the sources it runs (bench.src_hash()), i.e. the
capture is of the benched tree.  --src-hash: the hash printed on the GPU box
at capture time (default: this tree's).
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

UNITS = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1, "ms": 1, "s": 1e3, "second": 1e3}

FIELDS = {
    "ms": ("gpu__time_duration.sum", "time"),
    "dram_read_bytes": ("dram__bytes_read.sum", "bytes"),
    "dram_write_bytes": ("dram__bytes_write.sum", "bytes"),
    "lts_sectors": ("lts__t_sectors.sum", "num"),
    "l2_hit_pct": ("lts__t_sector_hit_rate.pct", "num"),
    "l1_hit_pct": ("l1tex__t_sector_hit_rate.pct", "num"),
    "dram_pct": ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "num"),
    "l2_pct": ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "num"),
    "l1tex_pct": ("l1tex__throughput.avg.pct_of_peak_sustained_active", "num"),
    "issue_pct": ("smsp__issue_active.avg.pct_of_peak_sustained_active", "num"),
    "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", "num"),
    "inst_executed": ("smsp__inst_executed.sum", "num"),
    "smem_wavefronts": ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "num"),
    "smem_bank_conflicts": ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "num"),
    "global_ld_requests": ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "num"),
    "global_ld_sectors": ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "num"),
    "long_scoreboard": ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "num"),
    "sm_cycles_min": ("sm__cycles_active.min", "num"),
    "sm_cycles_avg": ("sm__cycles_active.avg", "num"),
    "sm_cycles_max": ("sm__cycles_active.max", "num"),
    "registers": ("launch__registers_per_thread", "num"),
    "grid": ("launch__grid_size", "num"),
    "block": ("launch__block_size", "num"),
}


def rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return r[0], r[1], r[2:]


def num(v):
    return float(v.replace(",", "")) if v not in ("", "n/a") else None


def kernel_metrics(hdr, units, v):
    d = {}
    for key, (name, kind) in FIELDS.items():
        if name not in hdr:
            continue
        x = num(v[hdr.index(name)])
        if x is None:
            continue
        u = units[hdr.index(name)]
        if kind in ("bytes", "time"):
            x *= UNITS.get(u, 1)
        d[key] = x
    if "dram_read_bytes" in d:
        d["dram_bytes"] = d["dram_read_bytes"] + d.get("dram_write_bytes", 0.0)
        d["dram_gbs"] = d["dram_bytes"] / (d["ms"] / 1e3) / 1e9
    if "lts_sectors" in d:
        d["lts_bytes"] = 32 * d["lts_sectors"]
        d["lts_gbs"] = d["lts_bytes"] / (d["ms"] / 1e3) / 1e9
    st = [(h.split("stalled_")[1].split("_per")[0], num(v[i])) for i, h in enumerate(hdr)
          if h.startswith("smsp__average_warps_issue_stalled") and h.endswith("per_issue_active.ratio")
          and num(v[i]) is not None]
    st.sort(key=lambda x: -x[1])
    d["top_stalls"] = st[:6]
    return d


def main():
    rep, tag = sys.argv[1], sys.argv[2]
    cfg = sys.argv[3] if len(sys.argv) > 3 and not sys.argv[3].startswith("--") else "C3"
    import bench
    h = bench.src_hash()
    if "--src-hash" in sys.argv:
        h = sys.argv[sys.argv.index("--src-hash") + 1]
    hdr, units, vals = rows(rep)
    kernels = {}
    for v in vals:
        name = v[hdr.index("Kernel Name")]
        short = "k_count_flat" if "k_count_flat" in name else ("k_count" if "k_count" in name else name[:40])
        kernels[short] = kernel_metrics(hdr, units, v)  # the last launch of each kernel wins
    head = subprocess.run(["git", "-C", ROOT, "rev-parse", "--short=12", "HEAD"], capture_output=True,
                          text=True).stdout.strip()
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    allsum = json.load(open(p)) if os.path.exists(p) else {}
    allsum[cfg] = {"src_hash": h, "tag": tag, "git_head_at_summary": head,
                   "what": "ncu --set full --clock-control none of one count step's kernels "
                           "(cold-cache replays; bytes and ratios, not times, are the evidence)",
                   "kernels": kernels}
    json.dump(allsum, open(p, "w"), indent=1, sort_keys=True)
    txt = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "ncu_summary.py"), rep],
                         capture_output=True, text=True).stdout
    lines = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "ncu_lines.py"), rep, "30"],
                           capture_output=True, text=True).stdout
    with open(os.path.join(ROOT, "profiles", f"{tag}_{cfg.lower()}_ncu.txt"), "w") as f:
        f.write(f"# {tag} {cfg}: ncu --set full --clock-control none, src_hash {h}\n")
        f.write(txt)
        f.write("\n# stall samples by source line\n")
        f.write(lines)
    print(json.dumps(allsum[cfg], indent=1)[:3000])


if __name__ == "__main__":
    main()
