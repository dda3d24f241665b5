"""The production kernel under the dynamic (claim-order) super-tile schedule (SAM_DYN=1, the NEXT-3
ablation switch): the knob is read once per process, so the checks run in a child
process with the variable set, element by element against the oracle on multi-round sizes."""
from __future__ import annotations

import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys
sys.path.insert(0, sys.argv[1])
import numpy as np, torch, oracle, synth
import paper_conf_pldi_malekiyb16_b200 as S
from tests.helpers import compare
bad = []
for name, k, s, n in [("i32", 1, 1, 3_000_017), ("i64", 2, 1, 2_000_003), ("i64", 4, 4, 2_500_001), ("i32", 8, 3, 1_000_003),
                      ("i64", 8, 8, 1_500_007), ("f64", 1, 2, 1_000_001), ("f32", 3, 1, 800_011), ("i32", 5, 7, 900_001)]:
    kind = "uniform" if name.startswith("i") else "small"
    x = synth.make(n, name, kind, seed=11 * k + s)
    for incl in (True, False):
        y = S.scan(torch.from_numpy(x).cuda(), k, s, incl)
        torch.cuda.synchronize()
        try:
            compare(name, x, y.cpu().numpy(), k, s, incl)
        except AssertionError as e:
            bad.append(str(e)[:200])
print("BAD" if bad else "OK", bad)
"""


def test_dynamic_claims_parity():
    env = dict(os.environ, SAM_DYN="1")
    r = subprocess.run([sys.executable, "-c", CHILD, ROOT], env=env, cwd=ROOT, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0, r.stderr[-2000:]
    assert r.stdout.strip().startswith("OK"), r.stdout[-2000:]
