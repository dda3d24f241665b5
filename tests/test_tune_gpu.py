"""The install-time autotune table (lib/sam_tune.txt via SAM_TUNE_FILE): entries are
applied per (type, order, tuple, size range), entries that do not match leave the built-in defaults,
and every tuned launch still equals the oracle."""
from __future__ import annotations

import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(table_text, tmp_path):
    f = tmp_path / "tune.txt"
    f.write_text(table_text)
    env = dict(os.environ, SAM_TUNE_FILE=str(f))
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "tune_driver.py")], capture_output=True, text=True,
                       env=env, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    return json.loads(r.stdout.strip().splitlines()[-1])


def test_tune_table_applied_and_exact(tmp_path):
    table = ("# comment line\n"
             "u64 2 1 20 23 1 6 1 2\n"       # i64 k=2 s=1 at 2^21.5: M=1, lag 6, windowed fold, landing on
             "u32 4 4 22 24 2 0 2 0\n"       # i32 k=4 s=4 at 2^22.3: M=2, default lag, value-parallel
             "u64 1 8 25 33 3 0 0 0\n")      # i64 k=1 s=8 at 2^20: range does not match -> defaults
    base = _run("", tmp_path)
    tuned = _run(table, tmp_path)
    for key in tuned:
        assert tuned[key]["ok"] and base[key]["ok"], key
    assert tuned["i64 k=2 s=1"]["M"] == 1 and tuned["i64 k=2 s=1"]["lag"] == 6 and tuned["i64 k=2 s=1"]["vfold"] == 0
    assert tuned["i32 k=4 s=4"]["M"] == 2 and tuned["i32 k=4 s=4"]["vfold"] == 1
    assert tuned["i64 k=1 s=8"] == base["i64 k=1 s=8"]
