"""compute-sanitizer over the hand-synchronised kernels (SURVEY.md §4/§5 race detection):
memcheck (out-of-bounds / misaligned accesses), racecheck (shared-memory hazards) and synccheck
(barrier misuse) on small launches of every tcgen05/TMA kernel family and a two-slot schedule
(tools/sanitize_nodes.py).  Only libduet's kernels are instrumented (kernel-name filter)."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool):
    cmd = [SAN, "--tool", tool, "--kernel-name", "kns=duet", "--error-exitcode", "99",
           sys.executable, os.path.join(ROOT, "tools", "sanitize_nodes.py")]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    out = r.stdout + r.stderr
    print(out[-3000:])
    if r.returncode != 0 and "closed on this pool" in out:
        # the GPU pool's compute-sanitizer wrapper refuses every run (it exits at once, nothing is
        # launched); the race / ordering evidence is then the stress and parity tests
        pytest.skip("compute-sanitizer closed on this GPU pool: " + out.strip()[:160])
    assert r.returncode == 0, out[-4000:]
    clean = ("ERROR SUMMARY: 0 errors" in out) or ("0 hazards displayed (0 errors, 0 warnings)" in out)
    assert clean, out[-4000:]
    for k in ("gemm", "rnn", "conv", "stem", "conv7", "c2"):
        assert f"{k} ok" in out
