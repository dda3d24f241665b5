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

import oracle
import synth
from tests.helpers import DT, compare, torch_dtype

pytestmark = pytest.mark.gpu

N_SWEEP = 40009  # prime: ragged for every s; >= 5 tiles for every s (largest tile: 7168 elements)


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


N_MULTI = 148 * 3 * 7168 * 3 + 4099  # > 3 super-tiles per CTA on 148 SMs for every (dtype, s)


def _multi_round_input(name, k, s):
    """Inputs for the multi-round parity grid.  Ints: full-range bits (wraparound).  Floats: signed
    values in [-1, 1) scaled by a power of two so the order-k partial sums stay finite (R9)."""
    if name in ("i32", "i64"):
        return synth.make(N_MULTI, name, "uniform", seed=synth.SEED_BASE + 4242 + 16 * k + s)
    x = synth.make(N_MULTI, name, "unif01", seed=synth.SEED_BASE + 4343 + 16 * k + s)
    x = (x * DT[name](2) - DT[name](1))
    # order-k growth ~ (n/s)^k / k!: keep max |y| far below the format's range
    scale = {"f32": 2.0 ** -(6 * k), "f64": 2.0 ** -(6 * k)}[name]
    return (x * DT[name](scale)).astype(DT[name])


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", [1, 3, 4, 8])
def test_multi_round_schedule(name, k, s):
    """The full carry schedule (hand-off of a CTA's own inclusive state across >= 3 rounds, multi-
    window folds of the P-1 aggregates in between) for every dtype x order x tuple class, inclusive
    and exclusive, element by element against the oracle."""
    x = _multi_round_input(name, k, s)
    for inclusive in (True, False):
        compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive)


@pytest.mark.parametrize("name", ["f32", "f64"])
@pytest.mark.parametrize("k", [1, 2])
@pytest.mark.parametrize("s", [1, 3, 4, 8])
def test_multi_round_float_exact(name, k, s):
    """Integer-valued +-1 inputs at the multi-round size: bit-exact wherever every partial sum of
    every association order is an integer below 2^24 / 2^53 (SURVEY §8(c) floats): order 1 via the
    per-lane prefix range, order 2 via the order-2 scan of |x|."""
    x = synth.make(N_MULTI, name, "pm1int", seed=synth.SEED_BASE + 4444 + 16 * k + s)
    lim = 2.0 ** (24 if name == "f32" else 53)
    if k == 1:
        ref = oracle.scan(x, 1, s, True)[0].astype(np.float64)
        exact = all((np.ptp(np.concatenate([[0.0], ref[m::s]])) < lim) for m in range(s))
    else:
        exact = float(oracle.scan(np.abs(x), k, s, True)[0].max()) < lim
    for inclusive in (True, False):
        compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive, exact_float=exact)


@pytest.mark.parametrize("grid", [1, 2, 7, 37, 100])
@pytest.mark.parametrize("name,k,s", [("i32", 1, 1), ("i64", 4, 4), ("i32", 8, 3), ("f64", 2, 8)])
def test_reduced_grid_fallback(grid, name, k, s):
    """The cooperative-launch fallback (not all SMs available): grids above `grid` are
    refused, the launch shrinks the grid and retries; SAM's schedule must be exact for any P."""
    S = sam()
    x = synth.make(1 << 21, name, "uniform" if name[0] == "i" else "small", seed=synth.SEED_BASE + grid + k)
    S.sam_debug_limit_grid(grid)
    try:
        for inclusive in (True, False):
            compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive)
    finally:
        S.sam_debug_limit_grid(0)


@pytest.mark.parametrize("name,k,s", [("i32", 1, 1), ("i64", 1, 1), ("i32", 4, 1), ("i64", 8, 1), ("i64", 4, 4),
                                      ("i32", 2, 3), ("i64", 1, 5), ("f64", 3, 8)])
def test_stress_random_delays(name, k, s):
    """Randomised delays at every pipeline hand-over (sam_debug_set_stress), 100 seeds: every run
    equals the oracle-checked result bit for bit (SURVEY §4 tier 5)."""
    S = sam()
    xn = synth.make(148 * 2 * 7168 + 999, name, "uniform" if name[0] == "i" else "small", seed=synth.SEED_BASE + 17)
    x = torch.from_numpy(xn).cuda()
    ref = S.scan(x, k, s, True)
    torch.cuda.synchronize()
    compare(name, xn, ref.cpu().numpy(), k, s, True)
    try:
        for seed in range(1, 101):
            S.sam_debug_set_stress(seed)
            y = S.scan(x, k, s, True)
            torch.cuda.synchronize()
            assert torch.equal(y.view(torch.uint8), ref.view(torch.uint8)), f"stress seed {seed} differs"
    finally:
        S.sam_debug_set_stress(0)


def test_explicit_workspace_and_graph_growth():
    """sam_scan_ws: caller-owned workspace (zero-filled once), no allocation or synchronisation in
    the call, so a graph can be captured for a LARGER n than any earlier call (the cached workspace
    would need a grow + sync there)."""
    S = sam()
    dc = S.SAM_I32
    nmax = 3_000_017
    wsb = S.sam_scan_workspace_size(dc, 3, 2, nmax)
    ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
    for n in (1000, 77777, nmax):
        xn = synth.make(n, "i32", "uniform", seed=n)
        x = torch.from_numpy(xn).cuda()
        y = torch.empty_like(x)
        S.sam_scan_ws(dc, 3, 2, True, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), n,
                      ctypes.c_void_p(ws.data_ptr()), wsb, S._stream_ptr())
        torch.cuda.synchronize()
        compare("i32", xn, y.cpu().numpy(), 3, 2, True)
    # capture on a fresh stream with the explicit workspace, never used on that stream before
    xn = synth.make(nmax, "i32", "uniform", seed=4)
    x = torch.from_numpy(xn).cuda()
    y = torch.empty_like(x)
    st = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        S.sam_scan_ws(dc, 3, 2, False, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), nmax,
                      ctypes.c_void_p(ws.data_ptr()), wsb, S._stream_ptr(st))
    for _ in range(5):
        y.zero_()
        g.replay()
    torch.cuda.synchronize()
    compare("i32", xn, y.cpu().numpy(), 3, 2, False)


def test_epoch_wraparound_resets_carry_words():
    """the launch epoch in the carry tags wraps.  Tags are [20-bit epoch | 12-bit ring lap]
    with the epoch part cycling 1..2^20-1; put the epoch two launches before a restart and fill the
    carry ring with words carrying the tags the launches AFTER the restart will use (what launches
    2^20-1 earlier would have left): the restart launch zeroes the ring first, so none validates."""
    S = sam()
    dc = S.SAM_I64
    n = 1 << 21
    wsb = S.sam_scan_workspace_size(dc, 2, 3, n)
    ws = torch.zeros(wsb // 8, dtype=torch.int64, device="cuda")
    carry = ws[1024 // 8:]
    stale = torch.randint(0, 1 << 31, (carry.numel(),), dtype=torch.int64, device="cuda")
    ep_part = torch.randint(2, 5, (carry.numel(),), dtype=torch.int64, device="cuda")  # epochs 2..4, lap 0
    carry.copy_(stale | ((ep_part << 12) << 32))
    hdr32 = ws[:4].view(torch.int32)
    period = (1 << 20) - 1
    e0 = 5 * period - 2
    hdr32[3] = e0  # epoch word (offset 12): tags 2^20-2, 2^20-1, then the restart (reset, 1), 2, 3, 4
    xn = synth.make(n, "i64", "uniform", seed=123)
    x = torch.from_numpy(xn).cuda()
    for it in range(6):
        y = torch.empty_like(x)
        S.sam_scan_ws(dc, 2, 3, True, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), n,
                      ctypes.c_void_p(ws.data_ptr()), wsb, S._stream_ptr())
        torch.cuda.synchronize()
        compare("i64", xn, y.cpu().numpy(), 2, 3, True)
    assert int(hdr32[3].item()) == e0 + 6


@pytest.mark.parametrize("name,k,s", [("f32", 1, 1), ("f64", 1, 1), ("f32", 2, 3), ("f64", 4, 4)])
def test_float_bit_deterministic(name, k, s):
    # fixed association order (static carry schedule): identical bits run to run (R6)
    S = sam()
    x = torch.from_numpy(synth.make(1 << 24, name, "unif01", seed=synth.SEED_BASE + 99 + k + s)).cuda()
    y0 = S.scan(x, order=k, tuple=s, inclusive=True)
    for _ in range(3):
        y1 = S.scan(x, order=k, tuple=s, inclusive=True)
        assert torch.equal(y0.view(torch.uint8), y1.view(torch.uint8))


@pytest.mark.parametrize("teams", [1])
@pytest.mark.parametrize("land,vfold", [(1, 1), (1, 0), (0, 0)])
@pytest.mark.parametrize("name,k,s", [("i32", 1, 1), ("i64", 2, 1), ("i64", 4, 4), ("i32", 8, 3), ("f64", 3, 2),
                                      ("i64", 8, 8)])
def test_carry_team_variants(teams, land, vfold, name, k, s):
    """Every carry-pipeline variant (landing-buffer or windowed folds;
    value-parallel or windowed integer folds; odd tuples that make the ring records padded) over the
    multi-round schedule, against the oracle."""
    S = sam()
    x = _multi_round_input(name, k, s)
    S.sam_tune_override(-1, -1, vfold, land, teams)
    try:
        for inclusive in (True, False):
            compare(name, x, run(name, x, k, s, inclusive), k, s, inclusive)
    finally:
        S.sam_tune_override(-1, -1, -1, -1, -1)
