#!/usr/bin/env python
"""bench.py — oriented edges/s and TC ms of the ITC hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl b200tc|reference]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...

One "step" = one pass of the whole counting path over
the built graph of the workload: every rank counts its cost-balanced range of
live oriented edges (tc_count_range) and, for N > 1, one 8-byte NCCL
all_reduce combines the partials.  Preprocessing (a1-a6, tc_build_csr) is
timed separately and reported under "build_ms"; "e2e" times the public entry
point from pinned HOST edge lists: H2D copy + build + count + D2H of T.

Default workload: config C3 (RMAT scale 24, edge factor 16, Graph500
initiator, seed 1), the largest single-GPU RMAT graph BASELINE.json quotes the
metric on.  Inputs (1.1 GB CSR) exceed L2, and L2 is additionally flushed
between timed steps by writing a 512 MiB buffer.

Rank 0 prints ONE JSON line.  The oracle (oracle/, CPU) runs only in the
cpu_baseline leg (rank 0, N = 1) and under --impl reference.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import tcgen  # noqa: E402

METRIC = "oriented edges/sec"
UNIT = "edges/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C3", choices=sorted(tcgen.CONFIGS))
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--impl", default="b200tc", choices=["b200tc", "reference"])
    ap.add_argument("--flush-mb", type=int, default=512)
    ap.add_argument("--e2e-steps", type=int, default=None, help="default: --steps")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-e2e-pipelined", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0,
                    help="target oracle counting time of the cpu_baseline sample")
    ap.add_argument("--chunk-cost", type=int, default=0)
    ap.add_argument("--block", type=int, default=0)
    ap.add_argument("--opt", action="append", default=[],
                    help="plan option key=value (tc_options field), repeatable")
    ap.add_argument("--out", default=None, help="also write the JSON line here")
    ap.add_argument("--variant", default=None, choices=["polak", "trust"],
                    help="count with one of the paper's surveyed kernels (tc_count_variant, "
                         "SURVEY.md §8(f) f3) instead of the grouped path; N = 1 only")
    ap.add_argument("--reduce", default="nccl", choices=["nccl", "fused"],
                    help="cross-GPU sum of the partial counts: NCCL all_reduce, or the library's "
                         "own over NVLink peer memory (tc_count_range_fused, SURVEY.md §8(f) f4)")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for N > 1 (gloo: test mode only)")
    ap.add_argument("--share-gpu", action="store_true",
                    help="test mode: all ranks on cuda:0 with --backend gloo (exercises the N > 1 "
                         "code path on a one-GPU box; its timings are not scaling numbers)")
    ap.add_argument("--no-balance", action="store_true",
                    help="skip the N = 1 emulated multi-GPU balance measurement")
    ap.add_argument("--no-sharded", action="store_true",
                    help="skip the sharded-build measurement (tc_shard_*, SURVEY.md §8(f) f2)")
    ap.add_argument("--mode", default="count", choices=["count", "support"],
                    help="count: T (the headline); support: per-edge triangle counts "
                         "(tc_support, SURVEY.md §8(f) f1), N = 1 only")
    return ap.parse_args()


def cpu_info():
    model = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return model, os.cpu_count()


def expected_counts(cfg, seed):
    p = os.path.join(ROOT, "tests", "golden", "config_counts.json")
    if not os.path.exists(p):
        return None
    return json.load(open(p)).get(f"{cfg}/seed{seed}")


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


SRC_GLOBS = ("paper_conf_ipps_li0ptz24_b200/csrc", "include", "Makefile")


def src_hash():
    """sha256 (16 hex) over the sources that make libtc.so: the key that ties a
    committed ncu capture (profiles/ncu_summary.json) to the benched tree."""
    import hashlib
    h = hashlib.sha256()
    files = []
    for g in SRC_GLOBS:
        p = os.path.join(ROOT, g)
        if os.path.isdir(p):
            files += [os.path.join(p, f) for f in sorted(os.listdir(p))
                      if f.endswith((".cu", ".cuh", ".h"))]
        elif os.path.exists(p):
            files.append(p)
    for f in files:
        h.update(os.path.relpath(f, ROOT).encode())
        h.update(open(f, "rb").read())
    return h.hexdigest()[:16]


def profile_kernel(cfg, kernel):
    """ncu counters of `kernel` for this config from the committed summary, or
    (None, why) when it was not captured from these exact sources."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None, "no profiles/ncu_summary.json"
    d = json.load(open(p)).get(cfg)
    if not d or "kernels" not in d:
        return None, f"no capture for {cfg}"
    if d.get("src_hash") != src_hash():
        return None, f"capture {d.get('tag')} is of other sources ({d.get('src_hash')} != {src_hash()})"
    k = d["kernels"].get(kernel)
    return (k, d.get("tag")) if k else (None, f"{kernel} not in capture {d.get('tag')}")


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms (B200_PROFILING.md)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                       "-lms", "200", "-i", str(self.index)],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except OSError:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        rows = [l.strip().split(", ") for l in open(self.f.name) if l.strip()]
        os.unlink(self.f.name)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            try:
                sm.append(float(r[1]))
                mx.append(float(r[2]))
            except (ValueError, IndexError):
                continue
            for name, v in zip(names, r[5:9]):
                if v.strip() == "Active":
                    reasons.add(name)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(sm)}


def run_reference(a):
    """--impl reference: the CPU oracle, as it stands, on this box's host cores."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    cfg = tcgen.CONFIGS[a.config]
    tcgen.lib().tcgen_set_threads(0)
    src, dst, n = cfg.generate(a.seed)
    g = oracle.OracleGraph(src, dst, n)
    probe = g.count_rows(stride=4096, offset=0)
    m = probe.m
    # each step: rows x % stride == step, sized to ~cpu_seconds / (W+K) * ... bounded
    per_step_s = max(1.0, min(10.0, 120.0 / max(1, a.steps + a.warmup)))
    rate = probe.merge_steps_counted / max(probe.count_ms / 1e3, 1e-6)  # merge steps / s
    want_steps = rate * per_step_s
    stride = int(max(1, min(1 << 20, probe.merge_steps_total // max(want_steps, 1))))
    for i in range(a.warmup):
        g.count_rows(stride=stride, offset=i % stride)
    edges, secs, counted, total = 0.0, 0.0, 0, probe.merge_steps_total
    for i in range(a.steps):
        r = g.count_rows(stride=stride, offset=(a.warmup + i) % stride)
        frac = r.merge_steps_counted / max(1, r.merge_steps_total)
        edges += m * frac
        secs += r.count_ms / 1e3
        counted += r.merge_steps_counted
    value = edges / secs if secs > 0 else 0.0
    model, ncpu = cpu_info()
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": a.gpus,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": secs * 1e3 / max(1, a.steps),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32",
        "data": "synthetic", "config": {"workload": f"{a.config}: {cfg.description}",
                                        "seed": a.seed, "n": n, "m": m},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": r.threads, "kind": "oracle",
                         "sample": (f"rows x % {stride} == o (one offset o per step) of the "
                                    f"{a.config} graph; {counted / max(1, total) / a.steps:.4%} "
                                    f"of its merge steps per step; CPU {model}, {ncpu} cpus; "
                                    f"oracle build {g.count_rows(stride=1 << 30).build_ms:.0f} ms "
                                    f"not in value")},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    if a.out:
        open(a.out, "w").write(json.dumps(line) + "\n")
    g.close()
    return 0


def cpu_baseline(src, dst, n, a, m_gpu):
    """The oracle timed on a bounded row sample of the same workload (rank 0, N = 1)."""
    import oracle
    g = oracle.OracleGraph(src, dst, n)
    probe = g.count_rows(stride=4096, offset=0)
    rate = probe.merge_steps_counted / max(probe.count_ms / 1e3, 1e-6)
    stride = int(max(1, min(1 << 20, probe.merge_steps_total // max(rate * a.cpu_seconds, 1))))
    r = g.count_rows(stride=stride, offset=1 % stride)
    frac = r.merge_steps_counted / max(1, r.merge_steps_total)
    value = r.m * frac / max(r.count_ms / 1e3, 1e-9)
    model, ncpu = cpu_info()
    out = {"value": value, "unit": UNIT, "cores": r.threads, "kind": "oracle",
           "sample": (f"rows x % {stride} == 1 of the same graph ({frac:.3%} of its "
                      f"{r.merge_steps_total:.3e} merge steps, {r.count_ms:.0f} ms); "
                      f"value = m * sampled fraction / count time; oracle build "
                      f"{r.build_ms:.0f} ms excluded like the GPU build; CPU {model}, {ncpu} cpus"),
           "oracle_build_ms": r.build_ms}
    g.close()
    assert r.m == m_gpu, (r.m, m_gpu)
    return out


def bench_support(a, tc, g, info, src, dst, n, gen_s, build_wall_ms, world, rank):
    """--mode support: one step = tc_support over the resident graph (all m
    per-edge counts, zero-init included).  Parity: sum = 3T and 4,000 sampled
    edges against the oracle's |N(a) ∩ N(b)| (cpu leg)."""
    import torch
    if world > 1:
        if rank == 0:
            print(json.dumps({"metric": METRIC + " (per-edge support)", "unavailable":
                              "support mode is single-GPU (replicas only)"}), flush=True)
        return 0
    m = int(info.m)
    stream = torch.cuda.current_stream()
    sup = torch.empty(max(m, 1), dtype=torch.int32, device="cuda")[:m]
    flush = torch.empty(a.flush_mb << 20, dtype=torch.uint8, device="cuda")
    for _ in range(max(1, a.warmup)):
        g.support(out=sup)
    torch.cuda.synchronize()
    sampler = ClockSampler(torch.cuda.current_device())
    sampler.start()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(a.steps)]
    for i in range(a.steps):
        flush.fill_(i & 0xFF)
        evs[i][0].record(stream)
        g.support(out=sup)
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    step_ms = [x.elapsed_time(y) for x, y in evs]
    ms = sum(step_ms) / a.steps
    total = int(sup.to(torch.int64).sum().item())
    T = g.count()
    exp = expected_counts(a.config, a.seed)
    parity = {"sum_is_3T": total == 3 * T,
              "T_vs_oracle": None if exp is None else exp["triangles"] == T}
    if not a.no_cpu_baseline:
        import oracle
        idx = torch.randint(0, m, (4000,), generator=torch.Generator().manual_seed(1)).cuda()
        u, v = g.edge_list()
        su, sv, ss = (x[idx].cpu().numpy() for x in (u, v, sup))
        og = oracle.SupportGraph(src, dst, n)
        t0 = time.perf_counter()
        want = og.pairs(su, sv)
        cpu_s = time.perf_counter() - t0
        og.close()
        parity["sampled_4000_vs_oracle"] = bool(np.array_equal(ss.view(np.uint32).astype(np.int64),
                                                               want))
        cpu = {"value": 4000 / max(cpu_s, 1e-9), "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": "4,000 random edges of the same graph, |N(a) ∩ N(b)| one by one "
                         "(oracle SupportGraph.pairs, 1 thread); build excluded"}
    else:
        cpu = None
    hbm, peak_src = peaks()
    # the count's method bytes + the zeroed output + a 4-B read-modify-write for
    # each of the 3 edges of every triangle (random u32 atomics in L2: 3T of them)
    b = int(info.method_bytes) + 4 * m + 24 * T
    achieved = b / (ms / 1e3) / 1e9
    line = {
        "metric": METRIC + " (per-edge support)", "value": m / (ms / 1e3), "unit": UNIT,
        "n_gpus": 1, "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32",
        "data": "synthetic",
        "config": {"workload": f"{a.config}: {cfg_desc(a.config)}", "seed": a.seed, "n": n,
                   "m": m, "m_live": int(info.m_live), "mode": "support",
                   "l2": f"flushed by a {a.flush_mb} MiB write between timed steps"},
        "triangles": str(T), "parity_vs_oracle": parity,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                     "frac": achieved / hbm, "traffic": None, "bytes_per_launch": b,
                     "kernel": "k_support (both classes)", "kernel_ms": ms,
                     "bytes_def": "method bytes (tc_graph_info.method_bytes) + 4m (zero-init) + "
                                  "24T (3 u32 read-modify-writes per triangle)",
                     "atomics_per_s": 3 * T / (ms / 1e3),
                     "note": "bound by the L2's random u32 atomics (3 per triangle, the (u,v) ones "
                             "aggregated per tile run in the long class)",
                     "peak_source": peak_src},
        "gpu_launches": a.steps * 2,
        "build_ms": {"wall": build_wall_ms, "total_events": info.ms_total},
        "clocks": clocks, "gen_s": round(gen_s, 2), "step_ms": step_ms,
    }
    if cpu:
        line["cpu_baseline"] = cpu
    print(json.dumps(line), flush=True)
    if a.out:
        open(a.out, "w").write(json.dumps(line) + "\n")
    g.close()
    return 0


def cfg_desc(name):
    return tcgen.CONFIGS[name].description


def main():
    a = parse()
    if a.impl == "reference":
        return run_reference(a)

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_li0ptz24_b200 as tc

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != a.gpus and rank == 0:
        print(f"warning: --gpus {a.gpus} but WORLD_SIZE {world}", file=sys.stderr)
    if a.share_gpu:  # test mode: every rank on cuda:0 (gloo), to exercise the N > 1 path on one GPU
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if a.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(a.backend)
    dev = torch.device("cuda", local)

    cfg = tcgen.CONFIGS[a.config]
    tcgen.lib().tcgen_set_threads(0)
    t0 = time.time()
    src, dst, n = cfg.generate(a.seed)
    gen_s = time.time() - t0
    opts = {}
    if a.chunk_cost:
        opts["chunk_cost"] = a.chunk_cost
    if a.block:
        opts["block_threads"] = a.block
    # plan options: --opt k=v (repeatable) and BENCH_OPT="k=v,k=v" (for A/B drivers)
    for kv in a.opt + [x for x in os.environ.get("BENCH_OPT", "").split(",") if x]:
        k, v = kv.split("=")
        opts[k] = int(v)

    # ---------------------------------------------------------------- build (a1..a6)
    dsrc = torch.from_numpy(src).to(dev)
    dst_t = torch.from_numpy(dst).to(dev)
    g = tc.build_csr(dsrc, dst_t, n, options=opts or None)   # warm (allocator pools, CUB)
    g.close()
    torch.cuda.synchronize()
    tb = time.perf_counter()
    g = tc.build_csr(dsrc, dst_t, n, options=opts or None)
    torch.cuda.synchronize()
    build_wall_ms = (time.perf_counter() - tb) * 1e3
    info = g.info
    del dsrc, dst_t
    m = int(info.m)

    if a.mode == "support":
        return bench_support(a, tc, g, info, src, dst, n, gen_s, build_wall_ms, world, rank)

    # cost-balanced ranges: at N > 1 every rank measures the plan's time
    # profile (tc_calibrate) and the ranks agree on its average (one all_reduce)
    profile = tc.agreed_profile(g) if world > 1 else None
    bounds = g.partition(world, profile) if profile is not None else g.partition(world)
    e0, e1 = bounds[rank], bounds[rank + 1]
    # the rank's range split at the class boundary: the long class is k_count
    # (a8), the short class k_count_flat (a7); the timed step is the product
    # call over the whole range, the roofline times each class's call alone
    mlong = int(info.m_live_long)
    l0, l1 = e0, max(e0, min(e1, mlong))
    s0, s1 = max(e0, min(e1, mlong)), e1
    out = torch.zeros(3, dtype=torch.int64, device=dev)
    flush = torch.empty(a.flush_mb << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    if a.variant and world > 1:
        raise SystemExit("--variant runs on one GPU")

    fused = tc.FusedSum() if a.reduce == "fused" and not a.variant else None
    split = fused is None and not a.variant

    def step():
        if a.variant:
            g.count_variant(a.variant, out=out[0:1])
        elif fused is not None:  # count + the library's own cross-GPU sum in the last CTA (f4)
            fused.count_range(g, e0, e1, out=out[0:1])
        else:  # the product call: this rank's whole range, both classes
            g.count_range(e0, e1, out=out[0:1])
        if world > 1 and fused is None:
            dist.all_reduce(out[0:1])

    for _ in range(max(1, a.warmup)):
        step()
    torch.cuda.synchronize()
    T = int(out[0].item()) & (2**64 - 1)

    sampler = ClockSampler(torch.cuda.current_device())
    sampler.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(a.steps)]
    for i in range(a.steps):
        flush.fill_(i & 0xFF)  # L2 flush between timed steps (outside the events)
        x0, x1 = evs[i]
        x0.record(stream)
        step()
        x1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [x0.elapsed_time(x1) for x0, x1 in evs]

    # The kernels alone, for the roofline: the same range as one call per class
    # (k_count, then k_count_flat), events between them, L2 flushed; right
    # after the timed steps, same count.
    long_ms, kern_ms = list(step_ms), list(step_ms)
    if split:
        kev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(a.steps)]
        for i in range(a.steps):
            flush.fill_(i & 0xFF)
            y0, ym, y1 = kev[i]
            y0.record(stream)
            g.count_range(l0, l1, out=out[1:2])
            ym.record(stream)
            g.count_range(s0, s1, out=out[2:3])
            y1.record(stream)
        torch.cuda.synchronize()
        long_ms = [y0.elapsed_time(ym) for y0, ym, _ in kev]
        kern_ms = [y0.elapsed_time(y1) for y0, _, y1 in kev]
        assert (int(out[1].item()) + int(out[2].item())) & (2**64 - 1) == T or world > 1
    clocks = sampler.stop()
    tot = torch.tensor([sum(step_ms), sum(kern_ms), sum(long_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    total_ms, kern_total_ms, long_total_ms = float(tot[0]), float(tot[1]), float(tot[2])
    ms_per_step = total_ms / a.steps
    value = m / (ms_per_step / 1e3)

    # ---------------------------------------------------------------- sharded build (f2)
    # Every rank holds the contiguous 1/world slice of the raw pairs and the
    # ranks build the identical replicated graph (tc_shard_* + NCCL
    # all_reduce / all_to_all / broadcast); wall time after a device sync,
    # max over ranks.  At N = 1 it runs the same steps without collectives.
    lo, hi = rank * len(src) // world, (rank + 1) * len(src) // world
    sharded = None
    if not a.no_sharded:
        s_dev = torch.from_numpy(src[lo:hi]).to(dev)
        d_dev = torch.from_numpy(dst[lo:hi]).to(dev)
        g3 = tc.build_csr_sharded(s_dev, d_dev, n, options=opts or None)  # warm
        g3.close()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        phases = {}
        t3 = time.perf_counter()
        g3 = tc.build_csr_sharded(s_dev, d_dev, n, options=opts or None, timings=phases)
        torch.cuda.synchronize()
        sh_ms = (time.perf_counter() - t3) * 1e3
        same = int(g3.m == m and g3.m_live == info.m_live and g3.info.b_itc == info.b_itc)
        g3.close()
        del s_dev, d_dev
        x = torch.tensor([sh_ms, float(1 - same)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(x, op=dist.ReduceOp.MAX)
        sharded = {"wall_ms": float(x[0]), "same_graph_as_full_build": bool(x[1] == 0),
                   "phases_ms_rank0": {k: round(v, 3) for k, v in phases.items()},
                   "pairs_per_rank": int(hi - lo),
                   "what": "build_csr_sharded: tc_shard_canon, key-range all_to_all, "
                           "tc_shard_unique + degree all_reduce, tc_rank_vertices, tc_shard_orient, "
                           "row-range all_to_all + tc_sort_keys, ordered all-gather, "
                           "tc_build_from_oriented (max over ranks)"}

    # ---------------------------------------------------------------- e2e (public API, host data)
    e2e = None
    if not a.no_e2e:
        k2 = a.e2e_steps if a.e2e_steps is not None else a.steps
        ps = torch.from_numpy(src).pin_memory()
        pd = torch.from_numpy(dst).pin_memory()
        ts = []
        detail = []  # per step: host ms of the build call, the partition, the count + D2H; build phase ms (events)
        n_chunks = 0
        for i in range(1 + k2):  # first one warms the pinned path
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            x0 = torch.cuda.Event(enable_timing=True)
            x1 = torch.cuda.Event(enable_timing=True)
            x0.record(stream)
            h0 = time.perf_counter()
            if world > 1:  # each rank copies and sorts only its slice (f2)
                g2 = tc.build_csr_sharded(ps[lo:hi].to(dev, non_blocking=True),
                                          pd[lo:hi].to(dev, non_blocking=True), n,
                                          options=opts or None)
            else:
                g2 = tc.build_csr_host(ps, pd, n, options=opts or None)
            h1 = time.perf_counter()
            b = g2.partition(world, profile) if profile is not None else g2.partition(world)
            h2 = time.perf_counter()
            o2 = g2.count_range(b[rank], b[rank + 1])
            if world > 1:
                dist.all_reduce(o2)
            t_e2e = int(o2.item()) & (2**64 - 1)
            h3 = time.perf_counter()
            x1.record(stream)
            torch.cuda.synchronize()
            inf2 = g2.info
            n_chunks = inf2.n_chunks
            phases = [round(x, 1) for x in (inf2.ms_canon, inf2.ms_sort_unique, inf2.ms_degree_rank,
                                             inf2.ms_orient_csr, inf2.ms_plan, inf2.ms_total)]
            g2.close()
            assert t_e2e == T, (t_e2e, T)
            if i:
                ts.append(x0.elapsed_time(x1))
                detail.append([round(1e3 * (h1 - h0), 1), round(1e3 * (h2 - h1), 1), round(1e3 * (h3 - h2), 1),
                               phases])
        et = torch.tensor([sum(ts)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
        e2e_ms = float(et[0]) / max(1, len(ts))
        e2e = {"value": m / (e2e_ms / 1e3), "unit": UNIT, "ms_per_step": e2e_ms,
               "step_ms": [round(x, 3) for x in ts],
               "step_host_ms_build_partition_count": detail,
               "h2d_bytes_per_step": int(src.nbytes + dst.nbytes) * (hi - lo) // max(1, len(src)),
               "d2h_bytes_per_step": 8 + 8 * (n_chunks + 1) + 96,
               "what": ("tc_build_csr_host (H2D of the raw pinned edge list + a1..a6)" if world == 1
                        else "H2D of this rank's 1/N pinned slice + build_csr_sharded (f2)")
                       + " + tc_count_range + all_reduce + 8-B D2H of T"}

    # ---------------------------------------------------------------- e2e, pipelined over steps
    # The same public calls, but step i+1's H2D copy + build (tc_build_csr_host
    # on its own stream, in a second host thread: ctypes releases the GIL)
    # overlaps step i's count + D2H (another stream): the throughput of a
    # stream of graphs.  Reported next to "e2e" (one step at a time), which
    # stays the headline.  Host wall clock between two device syncs (the work
    # spans two streams and two threads).
    e2e_pipe = None
    if not a.no_e2e and world == 1 and not a.no_e2e_pipelined:
        import concurrent.futures
        k3 = a.e2e_steps if a.e2e_steps is not None else a.steps
        s_build, s_count = torch.cuda.Stream(), torch.cuda.Stream()

        def build_one():
            with torch.cuda.stream(s_build):
                return tc.build_csr_host(ps, pd, n, options=opts or None, stream=s_build)

        with concurrent.futures.ThreadPoolExecutor(1) as pool:
            for rep in range(2):  # the first pass warms both streams
                torch.cuda.synchronize()
                w0 = time.perf_counter()
                fut = pool.submit(build_one)
                for i in range(k3):
                    g3 = fut.result()
                    if i + 1 < k3:
                        fut = pool.submit(build_one)
                    t3 = g3.count(stream=s_count)  # count + 8-B D2H of T
                    g3.close()
                    assert t3 == T, (t3, T)
                torch.cuda.synchronize()
                wall = (time.perf_counter() - w0) * 1e3
        pipe_ms = wall / max(1, k3)
        e2e_pipe = {"value": m / (pipe_ms / 1e3), "unit": UNIT, "ms_per_step": pipe_ms, "steps": k3,
                    "h2d_bytes_per_step": int(src.nbytes + dst.nbytes), "d2h_bytes_per_step": 8,
                    "what": "the e2e calls with step i+1's H2D + build (second stream, second host "
                            "thread) overlapping step i's count + D2H; host wall clock between device "
                            "syncs / steps"}

    # ---------------------------------------------------------------- emulated multi-GPU balance
    # (after the e2e leg: its many short launches perturbed the e2e timing
    # that followed them, 13.6 -> 37 ms at C5)
    # N = 1: the P-rank splits of tc_partition_measured (this device's
    # 64-slice profile refined for P, as agreed_profile does at N = P) and of
    # tc_partition (built-in profile), every range
    # timed alone (L2 flushed, median of 3): max/mean per P
    balance = None
    if world == 1 and not a.variant and not a.no_balance:
        w = g.calibrate()
        balance = {"profile_slices": len(w), "profile_ms_sum": float(w.sum()),
                   "what": "each rank's tc_count_range timed alone on this GPU (CUDA events, "
                           "L2 flushed, median of 3); max/mean over ranks"}
        tmp = torch.zeros(1, dtype=torch.int64, device=dev)

        def range_ms(b, e):
            ts = []
            for r in range(3):
                flush.fill_(r)
                y0, y1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                y0.record(stream)
                g.count_range(b, e, out=tmp)
                y1.record(stream)
                torch.cuda.synchronize()
                ts.append(y0.elapsed_time(y1))
            return statistics.median(ts), int(tmp.item())

        for P in (2, 4, 8):
            for label, bb in (("measured", g.partition(P, g.refine(P, w))), ("builtin", g.partition(P))):
                res = [range_ms(bb[r], bb[r + 1]) for r in range(P)]
                ms = [x for x, _ in res]
                balance[f"P{P}_{label}"] = {
                    "max_over_mean": max(ms) / (sum(ms) / P), "range_ms": [round(x, 3) for x in ms],
                    "partials_sum_to_T": (sum(p for _, p in res) & (2**64 - 1)) == T}

    if rank != 0:
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        return 0

    exp = expected_counts(a.config, a.seed)
    parity = None if exp is None else (exp["triangles"] == T and exp["m"] == m)

    hbm, peak_src = peaks()
    # Roofline of the dominant kernel, k_count (the long class, a8): the
    # method's own bytes (4 B per trimmed key + the plan
    # entries + N+(v) once per (chunk, group)) over its CUDA-event time in
    # the timed region.  For N > 1: this rank's share of the long class, by
    # the plan cost of its chunks.
    seg, cost = g.chunks()
    nl = int(info.n_long_chunks)
    share = 1.0
    if world > 1 and cost[nl] > 0:
        c0, c1 = (int(np.searchsorted(seg[:nl + 1], x, side="left")) for x in (l0, l1))
        share = float(cost[c1] - cost[c0]) / float(cost[nl])
    long_s = long_total_ms / a.steps / 1e3
    kern_s = kern_total_ms / a.steps / 1e3
    short_s = kern_s - long_s
    if split and long_s >= short_s:
        b_launch = float(info.method_bytes_long) * share
        kname, kdesc = "k_count", "k_count (long class, a8), timed alone between its events"
        k_s = long_s
    elif split:  # the short class dominates (C2, C5): k_count_flat
        sshare = 1.0
        if world > 1 and cost[-1] > cost[nl]:
            c0, c1 = (int(np.searchsorted(seg, x, side="left")) for x in (s0, s1))
            sshare = float(cost[max(c1, nl)] - cost[max(c0, nl)]) / float(cost[-1] - cost[nl])
        b_launch = float(info.method_bytes - info.method_bytes_long) * sshare
        kname, kdesc = "k_count_flat", "k_count_flat (short class, a7), timed alone between its events"
        k_s = short_s
    else:  # variant / fused: one call, whole-step bytes
        b_launch = float(info.method_bytes) * (share if world > 1 else 1.0)
        kname, kdesc = "k_count", "whole count step (variant or fused: one call)"
        k_s = kern_s
    achieved = b_launch / k_s / 1e9
    frac = achieved / hbm
    prof, why = profile_kernel(a.config, kname) if world == 1 and not a.variant else (None, "N>1 or variant")
    step_bytes = float(info.method_bytes) * (1.0 if world == 1 else (e1 - e0) / max(1, info.m_live))
    roof = {"bound": "hbm", "kernel": kdesc, "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": frac,
            "traffic": None if prof is None else prof["dram_bytes"] * share,
            "traffic_source": (f"ncu --set full, capture {why}, same sources (src_hash {src_hash()})"
                               if prof is not None else f"none: {why}"),
            "bytes_per_launch": b_launch, "kernel_ms": k_s * 1e3,
            "bytes_def": "method bytes of the kernel's class = 4*keys + 16 B plan entries per "
                         "live edge + (4*d+(v) + 28 B) per (chunk, group) + 36 B per chunk "
                         "(info.method_bytes_long, or method_bytes - method_bytes_long for the "
                         "short class); x this rank's cost share for N>1",
            "peak_source": peak_src,
            "step": {"bytes": step_bytes, "ms": ms_per_step,
                     "frac": step_bytes / (ms_per_step / 1e3) / 1e9 / hbm,
                     "what": "the timed step (the product call over both classes), whole-step "
                             "method bytes"},
            "merge_equiv": {"bytes": float(info.b_itc),
                            "frac": float(info.b_itc) / (ms_per_step / 1e3) / 1e9 / hbm,
                            "what": "B_ITC (SURVEY.md §8(d), both operand lists per edge): context "
                                    "only, not a roofline - this design reads N+(v) once per group"}}
    if prof is not None:
        roof["ncu"] = {k: prof.get(k) for k in ("dram_bytes", "lts_bytes", "l2_hit_pct", "l1_hit_pct",
                                                "dram_pct", "l1tex_pct", "issue_pct",
                                                "warps_active_pct", "long_scoreboard")}
    if frac > 1.2:
        raise SystemExit(f"roofline frac {frac:.2f} > 1.2: the bytes do not describe the timed kernel")
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
        "warmup": a.warmup, "ms_per_step": ms_per_step, "tc_ms": ms_per_step,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32",
        "data": "synthetic",
        "config": {"workload": f"{a.config}: {cfg.description}", "seed": a.seed, "n": n,
                   "n_active": int(info.n), "m": m, "max_out_degree": int(info.max_out_degree),
                   "m_live": int(info.m_live), "keys_total": int(info.keys_total),
                   "parallelism": f"edge-range x{world} (replicated CSR, " + (
                       "1 NCCL all_reduce)" if fused is None else
                       f"fused sum over NVLink peer memory, {fused.mode})"),
                   "l2": f"flushed by a {a.flush_mb} MiB write between timed steps; CSR "
                         f"{(info.m * 4 + (info.n + 1) * 8) / 2**20:.0f} MiB",
                   "kernel": a.variant or "grouped (k_count + k_count_flat)",
                   "src_hash": src_hash()},
        "triangles": str(T), "parity_vs_oracle": parity,
        "roofline": roof,
        "e2e": e2e,
        "e2e_pipelined": e2e_pipe,
        "emulated_balance": balance,
        "gpu_launches": a.steps * (((l1 > l0) + (s1 > s0) if split else g.launches_per_count)
                                   if not a.variant else (1 if a.variant == "polak" else 3)),
        "build_ms": {"canon": info.ms_canon, "sort_unique": info.ms_sort_unique,
                     "degree_rank": info.ms_degree_rank, "orient_csr": info.ms_orient_csr,
                     "plan": info.ms_plan, "total_events": info.ms_total,
                     "wall": build_wall_ms, "sharded": sharded},
        "plan": {"n_chunks": int(info.n_chunks), "grid": int(info.count_grid),
                 "block": int(info.count_block), "smem_bytes": int(info.smem_bytes),
                 "groups": int(info.n_groups)},
        "clocks": clocks,
        "gen_s": round(gen_s, 2),
        "step_ms": step_ms,
    }
    if world == 1 and not a.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(src, dst, n, a, m)
    print(json.dumps(line), flush=True)
    if a.out:
        open(a.out, "w").write(json.dumps(line) + "\n")
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
