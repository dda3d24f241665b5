"""Race / synchronisation checks (SURVEY §4 tier 5): the scan kernel under
compute-sanitizer's racecheck (shared-memory hazards between the producer, aggregator, carry and
compute warps), synccheck (barrier misuse) and memcheck, at small n for orders 1/4/8 and tuples
1/3/8, every result also compared with the oracle."""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["racecheck", "synccheck", "memcheck"])
def test_compute_sanitizer(tool):
    if not os.path.exists(SAN):
        pytest.skip("compute-sanitizer not found")
    cmd = [SAN, "--tool", tool, "--error-exitcode", "97", "--kernel-name", "kns=sam_scan_kernel",
           sys.executable, os.path.join(ROOT, "tests", "sanitize_driver.py")]
    if tool == "racecheck":
        cmd[3:3] = ["--racecheck-report", "hazard", "--print-limit", "400"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=3000, cwd=ROOT)
    out = r.stdout + r.stderr
    with open(os.path.join(ROOT, "gpurun_out", f"sanitizer_{tool}.txt") if os.path.isdir(os.path.join(ROOT, "gpurun_out")) else os.devnull, "w") as f:
        f.write(out)
    if "sanitize driver done" not in out and "closed on this pool" in out:
        # the pool's compute-sanitizer wrapper refuses to run (it has left GPUs needing a reset); the
        # round-2 clean runs are kept in profiles/r2_sanitizer_*.txt, the randomized-delay stress
        # tests (test_parity_gpu.py) cover the hand-overs in the meantime
        pytest.skip("compute-sanitizer is closed on this GPU pool")
    assert "sanitize driver done, mismatches: 0" in out, out[-3000:]
    assert r.returncode == 0, f"{tool} reported errors (exit {r.returncode}):\n{out[-3000:]}"
