"""bench.py contract checks that run without a GPU: the reference arm (the CPU oracle)
prints one JSON line with the keys the driver reads."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    import time
    t0 = time.perf_counter()
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "3", "--cpu-budget", "0.2", "--config", "cif"],
                         capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "frames/s"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["config"]["workload"] == "cif"
    # ms_per_step is a measured step (a bounded sample), so the timed steps fit in the run
    assert d["ms_per_step"] * d["steps"] / 1e3 <= time.perf_counter() - t0


def test_warmup_must_be_at_least_three():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--warmup", "2"],
                         capture_output=True, text=True, timeout=120, cwd=ROOT)
    assert out.returncode != 0


def test_workload_units_1080p():
    sys.path.insert(0, ROOT)
    import bench
    from synth import CONFIGS
    u = bench.workload_units(CONFIGS["1080p_sa64_4rf"])
    assert u["n_mb"] == 8160
    assert u["me_cands"] == 8160 * 4 * 4096 == 133_693_440     # 133.69 M MB-candidates
    assert u["me_px"] == 34_225_520_640                          # 34.23 G px-absdiffs
    assert u["sme_px"] == 8160 * 4 * 16 * 7 * 256                 # 0.936 G
    assert u["int_bytes"] == 16 * 1920 * 1088 == 33_423_360         # 16 B/px, 33.4 MB
