"""Sharded (multi-GPU) scan over contiguous shards, SURVEY §8(e).

One process per GPU.  Rank r holds elements [g_r, g_r + n_r) of the global array (rank order).

    1. sam_shard_state   read-only pass over the local shard -> payload
                         [u64 n_r][u64 g_r][k*s values] = zero-seeded state of each global lane
                         at its last element in the shard (<= 16 + 512 bytes)
    2. all_gather        NCCL all_gather_into_tensor of the payloads over NVLink / NVSwitch
                         (the one exchange step of the path)
    3. sam_shard_scan    fold of the payloads of ranks < r with the carry operator
                         (M(L) s + v) into this shard's seed, then the seeded
                         single-pass scan (binomial fix-up fused into the carry application)

Sharded delta ENCODER: each rank needs the order*tuple elements before its
shard.  Every rank contributes the last min(n_r, 64) elements of its shard (TAIL = 64 >= max k*s)
and n_r to one all-gather; rank r's halo is the last k*s elements of the concatenated valid tails
of ranks < r (left-padded with zeros), then sam_delta_encode_halo encodes the shard.  Pure data
movement on the host side; the differencing runs in the library's kernel.

torch.distributed is plumbing only; every arithmetic step runs in libsam.so kernels.
"""
from __future__ import annotations

import ctypes

import torch
import torch.distributed as dist

from . import (SamError, _stream_ptr, delta_encode, dtype_code, sam_cyclic_fold, sam_scan_seeded,
               sam_shard_payload_bytes, sam_shard_scan, sam_shard_state)

TAIL = 64  # elements each rank contributes to the halo exchange (>= max order*tuple = 64)


def shard_offsets(n_local: int, group=None, device=None) -> tuple[int, int]:
    """(global offset of this rank's shard, global n) from an all-gather of the shard lengths."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    t = torch.tensor([n_local], dtype=torch.int64, device=device)
    allv = torch.empty(world, dtype=torch.int64, device=device)
    dist.all_gather_into_tensor(allv, t, group=group)
    lens = allv.tolist()
    return int(sum(lens[:rank])), int(sum(lens))


def _gather(t: torch.Tensor, group=None) -> torch.Tensor:
    """all_gather_into_tensor in rank order.  NCCL moves CUDA tensors over NVLink; a gloo group
    (CPU tests, or several ranks sharing one GPU) gets the bytes staged through host memory."""
    world = dist.get_world_size(group)
    if t.is_cuda and dist.get_backend(group) == "gloo":
        h = t.cpu()
        out = torch.empty(world * h.numel(), dtype=h.dtype)
        dist.all_gather_into_tensor(out, h, group=group)
        return out.to(t.device, non_blocking=False)
    out = torch.empty(world * t.numel(), dtype=t.dtype, device=t.device)
    dist.all_gather_into_tensor(out, t, group=group)
    return out


def exchange_payloads(payload: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather the per-rank payloads (uint8) in rank order (NCCL over NVLink on GPUs)."""
    return _gather(payload, group)


def scan_sharded(x_local: torch.Tensor, order: int = 1, tuple: int = 1, inclusive: bool = True,
                 group=None, global_offset: int | None = None, out: torch.Tensor | None = None,
                 stream=None) -> torch.Tensor:
    """Scan of the global array whose contiguous shard `x_local` this rank holds.  Every step --
    state pass, all-gather, seeded scan -- is issued on `stream` (default: the current stream), so
    the collective is ordered after the payload it sends and before the scan that reads it."""
    if not x_local.is_cuda or x_local.dim() != 1 or not x_local.is_contiguous():
        raise SamError(-1, "x_local must be a 1-D contiguous CUDA tensor")
    st_obj = stream if stream is not None else torch.cuda.current_stream(x_local.device)
    with torch.cuda.stream(st_obj):
        world = dist.get_world_size(group)
        rank = dist.get_rank(group)
        if global_offset is None:
            global_offset, _ = shard_offsets(x_local.numel(), group, device=x_local.device)
        if out is None:
            out = torch.empty_like(x_local)
        dc = dtype_code(x_local.dtype)
        st = _stream_ptr(st_obj)
        n = x_local.numel()
        if world == 1:
            sam_shard_scan(dc, order, tuple, inclusive, ctypes.c_void_p(x_local.data_ptr()),
                           ctypes.c_void_p(out.data_ptr()), n, global_offset, None, 0, 1, st)
            return out
        pb = sam_shard_payload_bytes(dc, order, tuple)
        payload = torch.empty(pb, dtype=torch.uint8, device=x_local.device)
        sam_shard_state(dc, order, tuple, ctypes.c_void_p(x_local.data_ptr()), n, global_offset,
                        ctypes.c_void_p(payload.data_ptr()), st)
        gathered = exchange_payloads(payload, group)
        sam_shard_scan(dc, order, tuple, inclusive, ctypes.c_void_p(x_local.data_ptr()),
                       ctypes.c_void_p(out.data_ptr()), n, global_offset, ctypes.c_void_p(gathered.data_ptr()),
                       rank, world, st)
    return out


def scan_virtual_shards(x: torch.Tensor, bounds: list[int], order: int = 1, tuple: int = 1,
                        inclusive: bool = True) -> torch.Tensor:
    """Run the sharded schedule on ONE GPU over virtual shards x[bounds[i]:bounds[i+1]]
    (state pass per shard, payload concatenation in place of the all-gather, seeded scans).
    Exercises every multi-GPU code path except the NCCL transport."""
    dc = dtype_code(x.dtype)
    pb = sam_shard_payload_bytes(dc, order, tuple)
    p = len(bounds) - 1
    gathered = torch.empty(p * pb, dtype=torch.uint8, device=x.device)
    out = torch.empty_like(x)
    st = _stream_ptr()
    w = x.element_size()
    for r in range(p):
        lo, hi = bounds[r], bounds[r + 1]
        sam_shard_state(dc, order, tuple, ctypes.c_void_p(x.data_ptr() + lo * w), hi - lo, lo,
                        ctypes.c_void_p(gathered.data_ptr() + r * pb), st)
    for r in range(p):
        lo, hi = bounds[r], bounds[r + 1]
        sam_shard_scan(dc, order, tuple, inclusive, ctypes.c_void_p(x.data_ptr() + lo * w),
                       ctypes.c_void_p(out.data_ptr() + lo * w), hi - lo, lo,
                       ctypes.c_void_p(gathered.data_ptr()), r, p, st)
    return out


# ----------------------------------------------------------------------------- block-cyclic (NEXT-1)
# SAM's persistent-block carry scheme with the GPUs as the blocks.
# Chunk c (C elements, global offset c*C) lives on rank c mod p; round r = chunks r*p .. r*p+p-1.
# Per round a rank runs the state pass over its chunk (the chunk stays in L2), the p payloads of the
# round are exchanged, sam_cyclic_fold turns the round's base state + the payloads of ranks < rank
# into this chunk's seed (and the next round's base), and the seeded scan re-reads the chunk from
# L2: one HBM read and one write per element on every GPU (contiguous shards: 1.5x that).
def cyclic_chunks(n_total: int, chunk: int, nranks: int, rank: int) -> list[tuple[int, int, int]]:
    """This rank's chunks in round order: (global offset, length, offset in the local buffer)."""
    if chunk < 1 or nranks < 1 or not 0 <= rank < nranks:
        raise SamError(-1, "chunk >= 1 and 0 <= rank < nranks required")
    out, lo, r = [], 0, 0
    while (r * nranks + rank) * chunk < n_total:
        g0 = (r * nranks + rank) * chunk
        ln = min(chunk, n_total - g0)
        out.append((g0, ln, lo))
        lo += ln
        r += 1
    return out


def cyclic_rounds(n_total: int, chunk: int, nranks: int) -> int:
    """Rounds of the block-cyclic schedule (every rank takes part in every round; a rank without a
    chunk in the last round contributes an empty payload)."""
    return -(-(-(-n_total // chunk)) // nranks) if n_total > 0 else 0


def cyclic_local_len(n_total: int, chunk: int, nranks: int, rank: int) -> int:
    return sum(ln for _, ln, _ in cyclic_chunks(n_total, chunk, nranks, rank))


def to_cyclic(x: torch.Tensor, chunk: int, nranks: int, rank: int) -> torch.Tensor:
    """This rank's block-cyclic local buffer (its chunks concatenated) from a global array."""
    parts = [x[g0:g0 + ln] for g0, ln, _ in cyclic_chunks(x.numel(), chunk, nranks, rank)]
    return torch.cat(parts) if parts else x[:0].clone()


def from_cyclic(locals_: list, chunk: int, n_total: int) -> torch.Tensor:
    """Reassemble the global array from every rank's block-cyclic local buffer."""
    p = len(locals_)
    out = torch.empty(n_total, dtype=locals_[0].dtype, device=locals_[0].device)
    for g in range(p):
        for g0, ln, lo in cyclic_chunks(n_total, chunk, p, g):
            out[g0:g0 + ln] = locals_[g][lo:lo + ln]
    return out


def _cyclic_steps(x_local, out, order, tuple_, inclusive, chunk, n_total, rank, nranks, lookahead, st_obj,
                  seed=None):
    """The per-rank schedule as a generator.  It yields ("send", r, payload) once the state pass of
    round r is issued and ("recv", r) when the fold of round r needs the gathered payloads (the
    driver sends back a device tensor of nranks * payload_bytes, rank order).  The state passes run
    up to `lookahead` rounds ahead of the folds, so the exchange of round r overlaps the state pass
    of round r + 1 (at the price of lookahead + 1 chunks held in L2).  Every kernel goes on st_obj."""
    dc = dtype_code(x_local.dtype)
    pb = sam_shard_payload_bytes(dc, order, tuple_)
    dev = x_local.device
    w = x_local.element_size()
    chunks = cyclic_chunks(n_total, chunk, nranks, rank)
    R = cyclic_rounds(n_total, chunk, nranks)
    st = _stream_ptr(st_obj)
    nbuf = lookahead + 2
    payloads = torch.empty(nbuf, pb, dtype=torch.uint8, device=dev)
    k_s = order * tuple_
    base = torch.zeros(k_s, dtype=x_local.dtype, device=dev)
    if seed is not None:
        base.copy_(seed.reshape(-1))
    seedbuf = torch.empty(k_s, dtype=x_local.dtype, device=dev)
    xp, op_ = x_local.data_ptr(), out.data_ptr()

    def state(r):
        pl = payloads[r % nbuf]
        if r < len(chunks):
            g0, ln, lo = chunks[r]
        else:  # no chunk of this rank in round r: an empty payload (every lane passes through)
            g0, ln, lo = (r * nranks + rank) * chunk, 0, 0
        sam_shard_state(dc, order, tuple_, ctypes.c_void_p(xp + lo * w if ln else 0), ln, g0,
                        ctypes.c_void_p(pl.data_ptr()), st)
        return pl

    for r in range(min(lookahead + 1, R)):
        yield ("send", r, state(r))
    for r in range(R):
        gathered = yield ("recv", r)
        sam_cyclic_fold(dc, order, tuple_, ctypes.c_void_p(gathered.data_ptr()), rank, nranks,
                        ctypes.c_void_p(base.data_ptr()), ctypes.c_void_p(seedbuf.data_ptr()),
                        ctypes.c_void_p(base.data_ptr()), st)
        if r < len(chunks):
            g0, ln, lo = chunks[r]
            sam_scan_seeded(dc, order, tuple_, inclusive, ctypes.c_void_p(xp + lo * w),
                            ctypes.c_void_p(op_ + lo * w), ln, g0, ctypes.c_void_p(seedbuf.data_ptr()), None, st)
        if r + lookahead + 1 < R:
            yield ("send", r + lookahead + 1, state(r + lookahead + 1))


def scan_cyclic(x_local: torch.Tensor, order: int = 1, tuple: int = 1, inclusive: bool = True,
                chunk: int = 1 << 22, n_total: int | None = None, group=None, out: torch.Tensor | None = None,
                lookahead: int | None = None, stream=None) -> torch.Tensor:
    """Scan of a global array held block-cyclically: this rank's `x_local` is the concatenation of
    chunks rank, rank + p, rank + 2p, ... of `chunk` elements (to_cyclic).  One all-gather of p
    payloads (<= 528 B each) per round -- the exchange step -- issued asynchronously so it overlaps
    the next round's state pass; every arithmetic step runs in libsam.so kernels on `stream`."""
    if not x_local.is_cuda or x_local.dim() != 1 or not x_local.is_contiguous():
        raise SamError(-1, "x_local must be a 1-D contiguous CUDA tensor")
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    st_obj = stream if stream is not None else torch.cuda.current_stream(x_local.device)
    with torch.cuda.stream(st_obj):
        if n_total is None:
            t = torch.tensor([x_local.numel()], dtype=torch.int64, device=x_local.device)
            n_total = int(_gather(t, group).sum().item())
        if x_local.numel() != cyclic_local_len(n_total, chunk, world, rank):
            raise SamError(-1, "x_local does not hold this rank's block-cyclic chunks of n_total elements")
        if out is None:
            out = torch.empty_like(x_local)
        if lookahead is None:
            lookahead = 0 if world == 1 else 1
        gen = _cyclic_steps(x_local, out, order, tuple, inclusive, chunk, n_total, rank, world, lookahead, st_obj)
        nccl = dist.get_backend(group) == "nccl"
        pending = {}
        try:
            msg = next(gen)
            while True:
                if msg[0] == "send":
                    r, pl = msg[1], msg[2]
                    if world == 1:
                        pending[r] = (None, pl)
                    elif nccl:
                        g = torch.empty(world * pl.numel(), dtype=torch.uint8, device=pl.device)
                        pending[r] = (dist.all_gather_into_tensor(g, pl, group=group, async_op=True), g)
                    else:
                        pending[r] = (None, _gather(pl, group))
                    msg = gen.send(None)
                else:
                    work, g = pending.pop(msg[1])
                    if work is not None:
                        work.wait()  # the compute stream waits for the collective (not the host)
                    msg = gen.send(g)
        except StopIteration:
            pass
    return out


def scan_cyclic_virtual(x: torch.Tensor, nranks: int, chunk: int, order: int = 1, tuple: int = 1,
                        inclusive: bool = True, lookahead: int = 1) -> torch.Tensor:
    """The block-cyclic schedule of `nranks` virtual ranks on ONE GPU, in one process: each virtual
    rank runs the same per-rank generator as scan_cyclic over its to_cyclic buffer; the exchange
    is a concatenation once every rank has sent a round.  No kernel ever waits on another rank's
    kernel (all on one stream, in an order where every round's payloads exist before its folds)."""
    n = x.numel()
    st_obj = torch.cuda.current_stream(x.device)
    parts = [to_cyclic(x, chunk, nranks, g) for g in range(nranks)]
    outs = [torch.empty_like(pt) for pt in parts]
    gens = [_cyclic_steps(parts[g], outs[g], order, tuple, inclusive, chunk, n, g, nranks, lookahead, st_obj)
            for g in range(nranks)]
    sent: dict[int, list] = {}
    ready: dict[int, torch.Tensor] = {}
    msgs = [next(gen, None) for gen in gens]
    while any(m is not None for m in msgs):
        progress = False
        for g in range(nranks):
            while msgs[g] is not None:
                m = msgs[g]
                if m[0] == "send":
                    row = sent.setdefault(m[1], [None] * nranks)
                    row[g] = m[2].clone()
                    if all(v is not None for v in row):
                        ready[m[1]] = torch.cat(row)
                    reply = None
                elif m[1] in ready:
                    reply = ready[m[1]]
                else:
                    break
                try:
                    msgs[g] = gens[g].send(reply)
                except StopIteration:
                    msgs[g] = None
                progress = True
        if not progress:
            raise SamError(-5, "block-cyclic emulation made no progress")
    return from_cyclic(outs, chunk, n)


# ----------------------------------------------------------------------------- delta encoder
def shard_tail(x_local: torch.Tensor) -> torch.Tensor:
    """The last min(n, TAIL) elements of a shard, right-aligned in a zero tensor of TAIL."""
    t = torch.zeros(TAIL, dtype=x_local.dtype, device=x_local.device)
    m = min(x_local.numel(), TAIL)
    if m:
        t[TAIL - m:] = x_local[x_local.numel() - m:]
    return t


def halo_from_tails(tails: torch.Tensor, lens, rank: int, ks: int) -> torch.Tensor:
    """Halo of `rank` (the ks elements preceding its shard, zero-left-padded) from the gathered
    tails [world, TAIL] and shard lengths (a list, or an int64 tensor on the tails' device): the
    suffix of the valid tails of ranks < rank.  The valid tail of a shard is all of it when
    n < TAIL, so the concatenation ends with the last TAIL elements of the global prefix.  Pure
    tensor indexing, no host synchronisation."""
    if rank == 0:
        return torch.zeros(ks, dtype=tails.dtype, device=tails.device)
    lens_t = torch.as_tensor(lens, dtype=torch.int64, device=tails.device)[:rank]
    pos = torch.arange(TAIL, device=tails.device)
    valid = pos[None, :] >= (TAIL - torch.clamp(lens_t, max=TAIL))[:, None]  # [rank, TAIL]
    flat = tails[:rank].reshape(-1)
    v = valid.reshape(-1)
    # rc[i] = number of valid elements at or after i; the halo takes those with rc <= ks
    rc = torch.flip(torch.cumsum(torch.flip(v.to(torch.int64), [0]), 0), [0])
    take = v & (rc <= ks)
    dest = torch.where(take, ks - rc, torch.full_like(rc, ks))  # slot ks = discard
    halo = torch.zeros(ks + 1, dtype=tails.dtype, device=tails.device)
    halo.scatter_(0, dest, torch.where(take, flat, torch.zeros_like(flat)))
    return halo[:ks].contiguous()


def delta_encode_sharded(x_local: torch.Tensor, order: int = 1, tuple: int = 1, group=None,
                         out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Delta encoding (k-th order, stride s) of the global array whose contiguous shard `x_local`
    this rank holds: ONE all-gather of [n_r | shard tail] records, the halo assembled on the device
    (no host synchronisation), then sam_delta_encode_halo -- all on `stream`."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if world == 1:
        return delta_encode(x_local, order, tuple, out=out, stream=stream)
    st_obj = stream if stream is not None else torch.cuda.current_stream(x_local.device)
    with torch.cuda.stream(st_obj):
        w = x_local.element_size()
        rec = torch.empty(8 + TAIL * w, dtype=torch.uint8, device=x_local.device)
        rec[:8].view(torch.int64).fill_(x_local.numel())
        rec[8:].view(x_local.dtype).copy_(shard_tail(x_local))
        recs = _gather(rec, group).view(world, 8 + TAIL * w)
        lens_t = recs[:, :8].contiguous().view(torch.int64).reshape(world)
        tails = recs[:, 8:].contiguous().view(x_local.dtype).reshape(world, TAIL)
        halo = halo_from_tails(tails, lens_t, rank, order * tuple)
        return delta_encode(x_local, order, tuple, out=out, stream=st_obj, halo=halo)


def delta_virtual_shards(x: torch.Tensor, bounds: list[int], order: int = 1, tuple: int = 1) -> torch.Tensor:
    """The sharded encoder's schedule on ONE GPU over virtual shards x[bounds[i]:bounds[i+1]]
    (tail stacking in place of the all-gather)."""
    p = len(bounds) - 1
    shards = [x[bounds[r]:bounds[r + 1]] for r in range(p)]
    tails = torch.stack([shard_tail(sh) for sh in shards])
    lens = [sh.numel() for sh in shards]
    out = torch.empty_like(x)
    for r in range(p):
        if lens[r]:
            delta_encode(shards[r], order, tuple, out=out[bounds[r]:bounds[r + 1]],
                         halo=halo_from_tails(tails, lens, r, order * tuple))
    return out
