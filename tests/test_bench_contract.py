"""bench.py's JSON-line contract on CPU (-m "not gpu"): the reference arm
(--impl reference) runs the CPU oracle only, so its line can be checked here;
the GPU arm's line is produced on the B200 (profiles/rNN_bench_*.json)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_prints_one_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                        "--config", "C1", "--steps", "2", "--warmup", "1"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "config", "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["unit"] == d["unit"]
    assert d["config"]["workload"].startswith("C1")


def test_gpu_committed_bench_lines_carry_the_contract_keys():
    """The latest committed GPU bench line of the headline config (profiles/)."""
    p = os.path.join(ROOT, "profiles")
    tags = sorted(f for f in os.listdir(p) if f.endswith("_bench_c3.json") and f.startswith("r"))
    assert tags, "no committed C3 bench line"
    d = json.load(open(os.path.join(p, tags[-1])))
    for k in ("metric", "value", "unit", "n_gpus", "ms_per_step", "roofline", "cpu_baseline", "e2e",
              "gpu_launches", "clocks", "dtype", "config"):
        assert k in d, k
    rf = d["roofline"]
    assert rf["bound"] == "hbm" and rf["unit"] == "GB/s" and abs(rf["frac"] - rf["achieved"] / rf["peak"]) < 1e-9
    assert d["parity_vs_oracle"] is True and d["gpu_launches"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] > 0
