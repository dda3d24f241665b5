"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Integers bit-exact; floats within rtol*sqrt(n*k)*A (R7) plus exact checks on
integer-valued inputs.  Sizes span several tiles (T = 3328..7168 elements) and a ragged tail; the
multi-round sizes give every CTA several super-tiles, so the carry schedule's hand-off of a CTA's
own inclusive state and its multi-window folds of the P-1 aggregates in between are exercised.
"""
from __future__ import annotations

import ctypes

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import synth
from tests.helpers import DT, compare, torch_dtype

pytestmark = pytest.mark.gpu

N_SWEEP = 20011  # prime: ragged for every s, >= 5 tiles for every s


def sam():
    import paper_conf_pldi_malekiyb16_b200 as S

    return S


def run(name, x_np, k, s, inclusive, out=None):
    S = sam()
    x = torch.from_numpy(x_np).cuda()
    y = S.scan(x, order=k, tuple=s, inclusive=inclusive, out=out)
    torch.cuda.synchronize()
    return y.cpu().numpy()


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", range(1, 9))
def test_sweep_dtype_order_tuple(name, k, s):
    kind = "uniform" if name in ("i32", "i64") else ("unif01" if k <= 2 else "small")
    x = synth.make(N_SWEEP, name, kind, seed=synth.SEED_BASE + 1000 + 10 * k + s)
    if name in ("f32", "f64") and k > 2:
        x = x * DT[name](1.0 / 64)  # keep high orders finite (reading R9)
    for inclusive in (True, False):
        compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive)


@pytest.mark.parametrize("name", ["f32", "f64"])
@pytest.mark.parametrize("s", range(1, 9))
def test_float_integer_valued_exact(name, s):
    # pm1int partial sums stay far below 2^24: every association order is exact (SURVEY §8(c) floats)
    x = synth.make(300007, name, "pm1int", seed=synth.SEED_BASE + 77 + s)
    for k in (1, 2):
        for inclusive in (True, False):
            compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive, exact_float=(k == 1))


@pytest.mark.parametrize("name", ["i32", "i64"])
@pytest.mark.parametrize("k,s", [(1, 1), (2, 1), (8, 1), (1, 8), (4, 4), (3, 3), (8, 8), (5, 7), (2, 6)])
def test_deep_lookback_many_tiles(name, k, s):
    n = (1 << 21) + 12345  # ~550 tiles: look-back windows, INCL/AGG mixes, persistent loop
    x = synth.make(n, name, "uniform", seed=synth.SEED_BASE + 5 + k * 8 + s)
    for inclusive in (True, False):
        compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive)


def tile_elems(s, items):
    """Tile size of the kernel geometry: W*32*items, W = s' * c."""
    G = s & -s
    sp = s // G
    c = max(1, 8 // sp)
    while c & (c - 1):
        c &= c - 1
    return sp * c * 32 * items


@pytest.mark.parametrize("k,s", [(1, 1), (3, 2), (8, 8), (2, 5), (4, 3), (1, 7)])
def test_edge_sizes(k, s):
    from paper_conf_pldi_malekiyb16_b200 import tile_items
    for name, items in (("i32", tile_items("i32")), ("i64", tile_items("i64"))):
        T = tile_elems(s, items)
        for n in sorted({1, 2, 3, s - 1 if s > 1 else 1, s, s + 1, 31, 32, 33, T - 1, T, T + 1, 2 * T - 1,
                         2 * T + 3, 3 * T + 5, 7 * T + s}):
            x = synth.make(n, name, "uniform", seed=n)
            for inclusive in (True, False):
                compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive)


def test_n_zero_is_noop():
    S = sam()
    x = torch.empty(0, dtype=torch.int32, device="cuda")
    y = S.scan(x, 3, 2)
    assert y.numel() == 0


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
def test_in_place(name):
    S = sam()
    for k, s in ((1, 1), (4, 3), (8, 8)):
        xn = synth.make(123457, name, "small", seed=k + s)
        x = torch.from_numpy(xn).cuda()
        S.scan(x, k, s, True, out=x)
        torch.cuda.synchronize()
        compare(name, xn, x.cpu().numpy(), k, s, True)


@pytest.mark.parametrize("name", ["i32", "i64"])
@pytest.mark.parametrize("off_in,off_out", [(1, 1), (3, 3), (1, 0), (0, 3), (2, 5)])
def test_misaligned_views(name, off_in, off_out):
    # element-aligned but not 16-B aligned buffers; equal misalignment uses the bulk-store path,
    # different misalignment the striped-store path
    S = sam()
    n = 100003
    for k, s in ((1, 1), (2, 3), (5, 8)):
        xn = synth.make(n, name, "uniform", seed=off_in * 7 + off_out + k)
        xb = torch.zeros(n + 8, dtype=torch_dtype(name), device="cuda")
        yb = torch.zeros(n + 8, dtype=torch_dtype(name), device="cuda")
        xb[off_in:off_in + n] = torch.from_numpy(xn).cuda()
        y = yb[off_out:off_out + n]
        S.scan(xb[off_in:off_in + n], k, s, True, out=y)
        torch.cuda.synchronize()
        compare(name, xn, y.cpu().numpy(), k, s, True)
        # guard elements untouched
        yh = yb.cpu().numpy()
        assert not yh[:off_out].any() and not yh[off_out + n:].any()


def test_repeat_launches_reuse_workspace():
    # the kernel resets its own tile counter / epoch: many back-to-back calls stay correct
    S = sam()
    xn = synth.make(500009, "i64", "uniform", seed=99)
    x = torch.from_numpy(xn).cuda()
    ys = [S.scan(x, 2, 3) for _ in range(50)]
    torch.cuda.synchronize()
    ref = ys[0].cpu().numpy()
    compare("i64", xn, ref, 2, 3, True)
    for y in ys[1:]:
        assert torch.equal(y, ys[0])


def test_two_streams_concurrently():
    S = sam()
    xa = synth.make(1 << 20, "i32", "uniform", seed=1)
    xb = synth.make(1 << 20, "i32", "uniform", seed=2)
    ta, tb = torch.from_numpy(xa).cuda(), torch.from_numpy(xb).cuda()
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    with torch.cuda.stream(sa):
        ya = [S.scan(ta, 3, 1) for _ in range(5)]
    with torch.cuda.stream(sb):
        yb = [S.scan(tb, 3, 1) for _ in range(5)]
    torch.cuda.synchronize()
    compare("i32", xa, ya[-1].cpu().numpy(), 3, 1, True)
    compare("i32", xb, yb[-1].cpu().numpy(), 3, 1, True)


def test_cuda_graph_capture():
    S = sam()
    xn = synth.make(300001, "i32", "uniform", seed=5)
    x = torch.from_numpy(xn).cuda()
    y = torch.empty_like(x)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        S.scan(x, 2, 2, out=y)  # creates the workspace for this stream before capture
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        S.scan(x, 2, 2, out=y)
    for _ in range(3):
        y.zero_()
        g.replay()
    torch.cuda.synchronize()
    compare("i32", xn, y.cpu().numpy(), 2, 2, True)


def test_errors_raise():
    S = sam()
    x = torch.zeros(10, dtype=torch.int32, device="cuda")
    with pytest.raises(S.SamError):
        S.scan(x, 9, 1)
    with pytest.raises(S.SamError):
        S.scan(x, 1, 0)
    with pytest.raises(S.SamError):
        S.scan(torch.zeros(10, dtype=torch.int16, device="cuda"), 1, 1)
    big = torch.zeros(100, dtype=torch.int32, device="cuda")
    with pytest.raises(S.SamError):
        S.scan(big[:50], 1, 1, out=big[10:60])  # partial overlap


@pytest.mark.parametrize("name", ["i32", "f64"])
def test_scan_host_pipeline(name):
    S = sam()
    n = (100 << 20) + 17 if name == "i32" else (1 << 24) + 5  # i32: 4 chunks of 128 MiB
    xn = synth.make(n, name, "small", seed=3)
    x = torch.from_numpy(xn).pin_memory()
    for k, s in ((1, 1), (3, 4)):
        y = S.scan_host(x, k, s, True)
        compare(name, xn, y.numpy(), k, s, True)


@pytest.mark.parametrize("name,k,s", [("i32", 1, 1), ("i32", 2, 1), ("i32", 3, 1), ("i64", 1, 1), ("i64", 4, 1),
                                      ("i64", 1, 3), ("i64", 2, 8), ("i32", 8, 1), ("i64", 8, 5)])
def test_multi_round_schedule(name, k, s):
    # > 3 super-tiles per CTA on 148 SMs (tiles of 3328..7168 elements, super-tiles of 2-3 tiles)
    n = 148 * 3 * 7168 * 3 + 4099
    x = synth.make(n, name, "uniform", seed=synth.SEED_BASE + 4242 + 16 * k + s)
    for inclusive in (True, False):
        compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive)


@pytest.mark.parametrize("name,k,s", [("f32", 1, 1), ("f64", 1, 1), ("f32", 2, 3), ("f64", 4, 4)])
def test_float_bit_deterministic(name, k, s):
    # fixed association order (static carry schedule): identical bits run to run (R6)
    S = sam()
    x = torch.from_numpy(synth.make(1 << 24, name, "unif01", seed=synth.SEED_BASE + 99 + k + s)).cuda()
    y0 = S.scan(x, order=k, tuple=s, inclusive=True)
    for _ in range(3):
        y1 = S.scan(x, order=k, tuple=s, inclusive=True)
        assert torch.equal(y0.view(torch.uint8), y1.view(torch.uint8))
