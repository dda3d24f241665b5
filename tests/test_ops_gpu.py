"""GPU parity of the other operators (xor, max, min) and
of the carry-scheme ablation (NEXT-3: SAM's static schedule, decoupled look-back, chained;
P:2319-2365) through the C ABI, against the oracle element by element.  Integers bit-exact; max/min
floats bit-exact too (no rounding: every output is one of the inputs or the identity); add floats
within the R7 tolerance."""
from __future__ import annotations

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
import synth
from tests.helpers import compare

pytestmark = pytest.mark.gpu

NP = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "f32": np.float32, "f64": np.float64}


def _x(n, name, seed):
    base = synth.make(n, "i64" if name in ("i64", "u64") else "i32", "uniform", seed=seed)
    if name in ("f32", "f64"):
        x = (synth.make(n, name, "unif01", seed=seed) * 2000 - 1000).astype(NP[name])
        x[::97] = np.nan  # maxNum semantics: NaN operands ignored
        return x
    if name[0] == "u":
        return base.view(np.uint32 if name == "u32" else np.uint64)
    return base


def _t(x):
    if x.dtype == np.uint32:
        return torch.from_numpy(x.view(np.int32)).cuda().view(torch.uint32)
    if x.dtype == np.uint64:
        return torch.from_numpy(x.view(np.int64)).cuda().view(torch.uint64)
    return torch.from_numpy(x).cuda()


def _np(y, dt):
    if y.dtype == torch.uint32:
        return y.view(torch.int32).cpu().numpy().view(np.uint32)
    if y.dtype == torch.uint64:
        return y.view(torch.int64).cpu().numpy().view(np.uint64)
    return y.cpu().numpy()


def _run(x, op, k, s, incl, carry=None):
    import paper_conf_pldi_malekiyb16_b200 as S

    y = S.scan_op(_t(x), op, k, s, incl, carry=carry)
    torch.cuda.synchronize()
    return _np(y, x.dtype)


def _eq(a, b):
    if a.dtype.kind == "f":
        return np.array_equal(a, b, equal_nan=True)
    return np.array_equal(a, b)


N_OPS = 3 * 8192 + 1237  # several tiles (4096 / 2048 lane positions... per s) and a ragged tail


@pytest.mark.parametrize("name", ["i32", "u32", "i64", "u64", "f32", "f64"])
@pytest.mark.parametrize("op", ["max", "min"])
@pytest.mark.parametrize("k,s", [(1, 1), (2, 1), (8, 1), (1, 3), (3, 4), (5, 8), (1, 7)])
def test_maxmin_parity(name, op, k, s):
    x = _x(N_OPS, name, seed=k * 16 + s)
    for incl in (True, False):
        ref = oracle.scan_op(x, op, k, s, incl)[0]
        got = _run(x, op, k, s, incl)
        assert _eq(got, ref), f"{op} {name} k={k} s={s} incl={incl}"


@pytest.mark.parametrize("name", ["i32", "u32", "i64", "u64"])
@pytest.mark.parametrize("k,s", [(1, 1), (2, 1), (3, 1), (8, 1), (1, 4), (2, 3), (4, 8), (7, 5)])
def test_xor_parity(name, k, s):
    x = _x(N_OPS, name, seed=100 + k * 16 + s)
    for incl in (True, False):
        ref = oracle.scan_op(x, "xor", k, s, incl)[0]
        assert _eq(_run(x, "xor", k, s, incl), ref), f"xor {name} k={k} s={s} incl={incl}"


@pytest.mark.parametrize("carry", ["static", "lookback", "chained"])
@pytest.mark.parametrize("op,name,k,s", [("add", "i32", 1, 1), ("add", "i64", 4, 4), ("add", "i32", 8, 3),
                                         ("add", "f64", 2, 1), ("xor", "u64", 3, 2), ("max", "i32", 4, 1),
                                         ("min", "f32", 1, 8)])
def test_carry_schemes(carry, op, name, k, s):
    """The same generic kernel under each carry scheme gives the oracle's result (the ablation
    compares like with like)."""
    n = 300_007 if carry != "chained" else 60_013
    x = _x(n, name, seed=7 * k + s)
    if op == "add" and name[0] == "f":
        x = synth.make(n, name, "small", seed=3)
    for incl in (True, False):
        got = _run(x, op, k, s, incl, carry=carry)
        if op == "add":
            compare(name, x, got, k, s, incl)
        else:
            assert _eq(got, oracle.scan_op(x, op, k, s, incl)[0]), f"{carry} {op} {name} k={k} s={s} incl={incl}"


def test_many_tiles_and_fallback_report():
    import paper_conf_pldi_malekiyb16_b200 as S

    x = _x((1 << 22) + 12345, "i64", seed=9)
    for op in ("xor", "max"):
        got = _run(x, op, 2, 3, True)
        assert _eq(got, oracle.scan_op(x, op, 2, 3, True)[0])
        assert S.sam_last_carry_scheme() in (0, 1)


def test_op_errors():
    import paper_conf_pldi_malekiyb16_b200 as S

    xf = torch.zeros(10, dtype=torch.float32, device="cuda")
    with pytest.raises(S.SamError):
        S.scan_op(xf, "xor")
    with pytest.raises(S.SamError):
        S.scan_op(xf, "nand")
