"""Sharded path on ONE GPU: virtual shards (state pass, payload concatenation in place of the
NCCL all-gather, fold, seeded scan) must reproduce the unsharded scan bit for bit (ints) for
p = 1..8 uneven shards, including empty shards and lengths not divisible by s (SURVEY §4 tier 3)."""
from __future__ import annotations

import ctypes

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
import synth
from tests.helpers import compare

pytestmark = pytest.mark.gpu


def _bounds(n, p, seed):
    rng = np.random.default_rng(seed)
    cuts = sorted(rng.integers(0, n + 1, size=p - 1).tolist())
    if p >= 3:
        cuts[1] = cuts[0]  # an empty shard
    return [0] + cuts + [n]


@pytest.mark.parametrize("name", ["i32", "i64", "f64"])
@pytest.mark.parametrize("k,s", [(1, 1), (4, 4), (8, 8), (3, 5), (2, 7), (1, 6)])
@pytest.mark.parametrize("p", [1, 2, 3, 5, 8])
def test_virtual_shards_match_unsharded(name, k, s, p):
    import paper_conf_pldi_malekiyb16_b200 as S
    from paper_conf_pldi_malekiyb16_b200.dist import scan_virtual_shards

    n = 200003
    kind = "uniform" if name != "f64" else "pm1int"
    xn = synth.make(n, name, kind, seed=synth.SEED_BASE + 31 * p + 7 * k + s)
    x = torch.from_numpy(xn).cuda()
    b = _bounds(n, p, seed=p * 100 + k * 10 + s)
    for inclusive in (True, False):
        ys = scan_virtual_shards(x, b, k, s, inclusive)
        y1 = S.scan(x, k, s, inclusive)
        torch.cuda.synchronize()
        if name != "f64":
            assert torch.equal(ys, y1), f"sharded != unsharded for p={p} bounds={b}"
        compare(name, xn, ys.cpu().numpy(), k, s, inclusive, exact_float=(name == "f64" and k <= 2))


@pytest.mark.parametrize("k,s", [(4, 4), (2, 3), (8, 1)])
def test_shard_state_payload_against_oracle(k, s):
    import paper_conf_pldi_malekiyb16_b200 as S

    n, g = 77777, 12345
    xn = synth.make(n, "i64", "uniform", seed=k * s)
    x = torch.from_numpy(xn).cuda()
    pb = S.sam_shard_payload_bytes(S.SAM_I64, k, s)
    pay = torch.zeros(pb, dtype=torch.uint8, device="cuda")
    S.sam_shard_state(S.SAM_I64, k, s, ctypes.c_void_p(x.data_ptr()), n, g, ctypes.c_void_p(pay.data_ptr()))
    torch.cuda.synchronize()
    ph = pay.cpu().numpy()
    hdr = ph[:16].view(np.uint64)
    assert int(hdr[0]) == n and int(hdr[1]) == g
    state = ph[16:].view(np.uint64).reshape(s, k)
    _, run = oracle.scan(xn, k, s, True, phase=g % s)
    assert np.array_equal(state, run.reshape(k, s).T)


def test_seeded_scan_continues_a_stream():
    import paper_conf_pldi_malekiyb16_b200 as S

    k, s = 3, 3
    n = 50001
    xn = synth.make(2 * n, "i32", "uniform", seed=4)
    x = torch.from_numpy(xn).cuda()
    out = torch.empty_like(x)
    st = torch.zeros(s * k, dtype=torch.int32, device="cuda")
    st2 = torch.zeros(s * k, dtype=torch.int32, device="cuda")
    P = lambda t: ctypes.c_void_p(t.data_ptr())
    S.sam_scan_seeded(S.SAM_I32, k, s, 1, P(x), P(out), n, 0, None, P(st))
    S.sam_scan_seeded(S.SAM_I32, k, s, 1, ctypes.c_void_p(x.data_ptr() + 4 * n),
                      ctypes.c_void_p(out.data_ptr() + 4 * n), n, n, P(st), P(st2))
    torch.cuda.synchronize()
    compare("i32", xn, out.cpu().numpy(), k, s, True)
    _, run = oracle.scan(xn, k, s, True)
    assert np.array_equal(st2.cpu().numpy().view(np.uint32).reshape(s, k), run.reshape(k, s).T)


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
@pytest.mark.parametrize("k,s", [(1, 1), (2, 1), (3, 3), (4, 4), (5, 2), (8, 8), (7, 5), (6, 6)])
def test_state_kernel_payloads(name, k, s):
    """The dedicated state-pass kernel (sam_state.cuh): the payload of sam_shard_state against the
    oracle's running state, for n from 1 element to many tiles, global offsets with every lane
    phase, and base pointers off the 16-B grid (the bulk copies' aligned superset)."""
    import math

    import paper_conf_pldi_malekiyb16_b200 as S

    dc = {"i32": 0, "i64": 1, "f32": 2, "f64": 3}[name]
    pb = S.sam_shard_payload_bytes(dc, k, s)
    T = S.tile_items(name) * 256 if hasattr(S, "tile_items") else 3328
    for n, g, off in [(1, 0, 0), (5, 3, 1), (T - 1, 7, 0), (T + 1, 1, 3), (3 * T + 17, 0, 2), (100_003, 12345, 1),
                      (1_000_003, 5, 0)]:
        kind = "uniform" if name.startswith("i") else "small"
        xn = synth.make(n + 4, name, kind, seed=n + k * 8 + s)
        x = torch.from_numpy(xn).cuda()
        w = x.element_size()
        pay = torch.zeros(pb, dtype=torch.uint8, device="cuda")
        S.sam_shard_state(dc, k, s, ctypes.c_void_p(x.data_ptr() + off * w), n, g, ctypes.c_void_p(pay.data_ptr()))
        torch.cuda.synchronize()
        ph = pay.cpu().numpy()
        assert int(ph[:16].view(np.uint64)[0]) == n and int(ph[:16].view(np.uint64)[1]) == g
        seg = xn[off:off + n]
        _, run = oracle.scan(seg, k, s, True, phase=g % s)
        ref = run.reshape(k, s).T
        if name.startswith("i"):
            got = ph[16:16 + k * s * w].view(ref.dtype).reshape(s, k)
            assert np.array_equal(got, ref), f"n={n} g={g} off={off}"
        else:
            got = ph[16:16 + k * s * w].view(np.float32 if name == "f32" else np.float64).reshape(s, k).astype(np.float64)
            A = oracle.scan(np.abs(seg), k, s, True, phase=g % s)[1].reshape(k, s).T.astype(np.float64)
            tol = (1e-5 if name == "f32" else 1e-12) * math.sqrt(max(1, n) * k) * A
            assert (np.abs(got - ref.astype(np.float64)) <= tol).all(), f"n={n} g={g} off={off}"
