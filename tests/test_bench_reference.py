"""bench.py --impl reference (the oracle timed on the host cores): one JSON line
with the contract keys, bounded wall time."""
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_line():
    t0 = time.time()
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "c1",
                        "--steps", "40", "--warmup", "3", "--ref-seconds", "2"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 40 and d["warmup"] == 3
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    assert time.time() - t0 < 240


def test_roofline_work_counts():
    """bench.py's FLOP counts (SURVEY.md §8(d) units): the algorithmic count of each config's
    dominant kernel, and the executed count beside it (GRU's fourth gate block, 128-row batch tiles,
    E padded to 64) -- closed forms on the BASELINE.json shapes."""
    sys.path.insert(0, ROOT)
    import bench
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    c5, c4, c3, c2 = (W.build(c) for c in ("c5", "c4", "c3", "c2"))
    assert bench.node_work(c2, "fc1") == 2 * 2048 * 1664 * 1024 == bench.node_executed(c2, "fc1")
    assert bench.node_work(c5, "b4_gru") == 2 * 16 * 4096 * 3 * 1024 * (256 + 1024)
    assert bench.node_executed(c5, "b4_gru") * 3 == bench.node_work(c5, "b4_gru") * 4      # fourth gate block
    assert bench.node_work(c3, "lstmA") == bench.node_executed(c3, "lstmA") == 2 * 64 * 256 * 4 * 512 * (256 + 512)
    assert bench.node_executed(c4, "gru") == 2 * 64 * 128 * 4 * 1024 * (256 + 1024)         # B = 64 -> 128 rows
    assert bench.node_executed(c4, "gru") * 3 == bench.node_work(c4, "gru") * 8
