"""Multi-GPU genome-pair driver (one process per GPU, torch.distributed over NCCL / NVLink).

Seed extensions are independent ("the seeds can be partitioned easily"), so the only
collectives sit at the edges of the path:

1. rank ``src`` packs the two sequences to 2 bits per base on its GPU (``fastz_pack_sequence``) and broadcasts
   the packed words (+ N masks when present) and the seed list over NCCL; every rank builds its context from
   the packed device buffers (``fastz_create_packed``: reversed copies made on its own GPU);
2. seeds are permuted by a fixed low-discrepancy stride and cut into W contiguous shards (spreads the
   unknown-length long tail);
3. every rank runs the CUDA path on its shard (no communication);
4. per-rank record counts / CIGAR sizes are all-gathered, the device-resident records (64 B each) and CIGAR
   bytes are gathered to ``src`` over NCCL, and ``src`` restores seed order with index arithmetic on its GPU
   (scatter by seed index, exclusive scan of the CIGAR lengths, one gather of the text), then copies the result
   to the host once.

Results are byte-identical for any world size.  The collectives and the reassembly are plain torch tensor
plumbing (no per-record Python), so the same code runs on CPU tensors under ``gloo``: ``extend_fn`` can be
injected to test the host-side logic without a GPU (it then receives ASCII sequences, broadcast as bytes).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import fastz

REC_BYTES = 64  # fastz_alignment
_OFF_I64 = 6    # cigar_off: int64 word 6 of a record (byte 48)
_LEN_I32 = 14   # cigar_len: int32 word 14 of a record (byte 56)


def _stride(n: int) -> int:
    """An odd multiplier near n / golden ratio, coprime with n: k -> k * a mod n is a bijection of [0, n)."""
    import math
    a = max(1, int(n * 0.6180339887498949)) | 1
    while math.gcd(a, n) != 1:
        a += 2
    return a


def shard_order(n: int) -> np.ndarray:
    """Deterministic low-discrepancy permutation of seed indices (position k holds seed k * a mod n): each
    rank's contiguous range of it samples the whole seed list evenly, so the unknown-length long tail spreads."""
    if n == 0:
        return np.zeros(0, dtype=np.int64)
    return (np.arange(n, dtype=np.int64) * _stride(n)) % n


def shard_indices(n: int, world: int, rank: int) -> np.ndarray:
    """Seed indices of ``rank``'s shard (sorted): positions [n*rank/W, n*(rank+1)/W) of shard_order(n)."""
    lo = (n * rank) // world
    hi = (n * (rank + 1)) // world
    if hi <= lo:
        return np.zeros(0, dtype=np.int64)
    return np.sort((np.arange(lo, hi, dtype=np.int64) * _stride(n)) % n)


def _world(group=None):
    if not dist.is_available() or not dist.is_initialized():
        return 1, 0
    return dist.get_world_size(group), dist.get_rank(group)


def _dev(group=None) -> torch.device:
    if dist.is_initialized() and dist.get_backend(group) != "nccl":
        return torch.device("cpu")
    return torch.device("cuda", torch.cuda.current_device())


def _bcast(t: torch.Tensor, src: int, group=None) -> torch.Tensor:
    if _world(group)[0] > 1 and t.numel():
        dist.broadcast(t, src, group=group)
    return t


def broadcast_bytes(data: bytes | None, src: int = 0, group=None) -> bytes:
    """Host bytes from ``src`` to every rank (used for injected extend functions and small metadata)."""
    dev = _dev(group)
    world, rank = _world(group)
    n = torch.tensor([len(data) if rank == src else 0], dtype=torch.int64, device=dev)
    _bcast(n, src, group)
    if rank == src:
        buf = torch.frombuffer(bytearray(data), dtype=torch.uint8).to(dev) if len(data) else \
            torch.zeros(0, dtype=torch.uint8, device=dev)
    else:
        buf = torch.empty(int(n.item()), dtype=torch.uint8, device=dev)
    _bcast(buf, src, group)
    return bytes(buf.cpu().numpy().tobytes())


def _gather_var(t: torch.Tensor, src: int, group=None):
    """Gather variable-length uint8 tensors (same device) to ``src``: all_gather of sizes, padded gather.
    Returns the list of per-rank tensors on ``src``, None elsewhere."""
    world, rank = _world(group)
    if world == 1:
        return [t]
    dev = t.device
    sz = torch.tensor([t.numel()], dtype=torch.int64, device=dev)
    sizes = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(sizes, sz, group=group)
    sizes = [int(s.item()) for s in sizes]
    mx = max(max(sizes), 1)
    buf = torch.zeros(mx, dtype=torch.uint8, device=dev)
    buf[:t.numel()] = t
    if rank == src:
        bufs = [torch.empty(mx, dtype=torch.uint8, device=dev) for _ in range(world)]
        dist.gather(buf, bufs, dst=src, group=group)
        return [bufs[r][:sizes[r]] for r in range(world)]
    dist.gather(buf, None, dst=src, group=group)
    return None


def merge_shards(idx_parts, rec_parts, cig_parts, n: int):
    """Restore seed order from per-rank shards (tensors on one device; no per-record Python).

    idx_parts[r]: int64 seed indices of rank r's records; rec_parts[r]: uint8 [n_r, 64] records whose
    cigar_off points into cig_parts[r].  Returns (uint8 [n, 64] records in seed order with cigar_off rebased
    into the merged text, uint8 merged text)."""
    dev = rec_parts[0].device
    idx = torch.cat([p.to(torch.int64) for p in idx_parts])
    rec = torch.cat([p.reshape(-1, REC_BYTES) for p in rec_parts])
    cig = torch.cat(cig_parts) if cig_parts else torch.zeros(0, dtype=torch.uint8, device=dev)
    assert idx.numel() == n and rec.shape[0] == n
    counts = torch.tensor([p.numel() for p in idx_parts], dtype=torch.int64, device=dev)
    sizes = torch.tensor([p.numel() for p in cig_parts], dtype=torch.int64, device=dev)
    base = torch.cumsum(sizes, 0) - sizes                           # each rank's text offset in `cig`
    r64 = rec.view(torch.int64)
    src_off = r64[:, _OFF_I64] + torch.repeat_interleave(base, counts)
    lens = rec.view(torch.int32)[:, _LEN_I32].to(torch.int64)
    inv = torch.empty(n, dtype=torch.int64, device=dev)
    inv[idx] = torch.arange(n, dtype=torch.int64, device=dev)       # output position -> input row
    out = torch.index_select(r64, 0, inv)                           # rows as 8 x int64 (fast row gather)
    olen = lens[inv]
    ooff = torch.cumsum(olen, 0) - olen
    out[:, _OFF_I64] = ooff
    out = out.view(torch.uint8)
    total = int(olen.sum().item()) if n else 0
    if total:
        # output byte b of record k comes from cig[b + starts[k]]: a step function of b, built as the cumsum of
        # its jumps at the records' output offsets (index_add: empty records share an offset, jumps telescope)
        starts = src_off[inv] - ooff
        jump = torch.zeros(total + 1, dtype=torch.int64, device=dev)
        jump.index_add_(0, ooff, starts - torch.cat([starts.new_zeros(1), starts[:-1]]))
        src = torch.cumsum(jump[:total], 0)
        src += torch.arange(total, dtype=torch.int64, device=dev)
        text = cig[src]
    else:
        text = torch.zeros(0, dtype=torch.uint8, device=dev)
    return out, text


def gather_results(idx: np.ndarray, rec: np.ndarray, cigar: bytes, n: int, group=None, dst: int = 0):
    """Host-array front end of the gather + merge (used with injected extend functions): returns
    (ALIGN_DTYPE records, cigar bytes) in seed order on ``dst``, (None, None) elsewhere."""
    dev = _dev(group)
    ti = torch.from_numpy(np.ascontiguousarray(idx, dtype=np.int64)).to(dev)
    tr = torch.from_numpy(np.ascontiguousarray(rec).view(np.uint8).reshape(-1)).to(dev)
    tc = torch.frombuffer(bytearray(cigar), dtype=torch.uint8).to(dev) if cigar else \
        torch.zeros(0, dtype=torch.uint8, device=dev)
    pi = _gather_var(ti.view(torch.uint8), dst, group)
    pr = _gather_var(tr, dst, group)
    pc = _gather_var(tc, dst, group)
    if _world(group)[1] != dst:
        return None, None
    out, text = merge_shards([p.view(torch.int64) for p in pi], [p.view(-1, REC_BYTES) for p in pr], pc, n)
    return out.cpu().numpy().reshape(-1).view(fastz.ALIGN_DTYPE), bytes(text.cpu().numpy().tobytes())


def _broadcast_packed(seq, src: int, group, device: int, stream) -> fastz.PackedSequence:
    """Pack on ``src`` (2 bits per base + N mask), broadcast the words over NCCL, return every rank's copy."""
    world, rank = _world(group)
    dev = torch.device("cuda", device)
    meta = torch.zeros(2, dtype=torch.int64, device=dev)
    if rank == src:
        ps = fastz.PackedSequence.pack(seq, device=device, stream=stream)
        meta[0], meta[1] = ps.length, 1 if ps.nmask is not None else 0
    _bcast(meta, src, group)
    length, has_n = int(meta[0].item()), bool(meta[1].item())
    nw = (length + 15) // 16
    if rank != src:
        ps = fastz.PackedSequence(torch.empty(nw, dtype=torch.int32, device=dev),
                                  torch.empty(nw, dtype=torch.int16, device=dev) if has_n else None, length)
    _bcast(ps.words, src, group)
    if has_n:
        _bcast(ps.nmask, src, group)
    return ps


def extend_genome_pair(T: bytes | None, Q: bytes | None, seeds: np.ndarray | None, params=None, group=None,
                       extend_fn=None, src: int = 0, mark_redundant: bool = False, mark_fn=None, timings=None,
                       torch_alloc: bool = False):
    """Collective: every rank calls it; only ``src`` needs real inputs.  Returns (records, cigar) on ``src`` as
    host arrays (ALIGN_DTYPE, bytes) in seed order, (None, None) elsewhere.

    ``mark_redundant``: after the gather, ``src`` runs the redundant-alignment post-pass (NEXT-3, reading R14)
    over the WHOLE record set -- the marks depend on every record, so they cannot be taken per shard -- setting
    FLAG_REDUNDANT (``mark_fn(rec)`` on host records if given, else the CUDA post-pass on the device records).
    ``timings``: optional dict that receives per-phase seconds on this rank.  ``torch_alloc``: the context's
    device memory comes from PyTorch's caching allocator (a long-running driver reuses it across pairs)."""
    import time
    world, rank = _world(group)
    dev = _dev(group)
    t0 = time.perf_counter()
    # 1. sequences + seeds
    if extend_fn is None:
        device = torch.cuda.current_device()
        stream = torch.cuda.current_stream(device).cuda_stream
        pT = _broadcast_packed(T, src, group, device, stream)
        pQ = _broadcast_packed(Q, src, group, device, stream)
    else:
        T = broadcast_bytes(T, src, group)
        Q = broadcast_bytes(Q, src, group)
    ns = torch.zeros(1, dtype=torch.int64, device=dev)
    if rank == src:
        ns[0] = len(seeds)
    _bcast(ns, src, group)
    n = int(ns.item())
    sd = torch.from_numpy(np.ascontiguousarray(seeds, dtype=np.int64).reshape(-1, 2)).to(dev) if rank == src else \
        torch.empty((n, 2), dtype=torch.int64, device=dev)
    _bcast(sd, src, group)
    idx_np = shard_indices(n, world, rank)
    idx = torch.from_numpy(idx_np).to(dev)
    t1 = time.perf_counter()
    # 2. the CUDA path on this rank's shard
    if extend_fn is None:
        with fastz.Aligner(pT, pQ, params, device=device, stream=stream, torch_alloc=torch_alloc) as al:
            al.extend_only(sd[idx])
            rec, cig = al.results_device()
            rec, cig = rec.clone(), cig.clone()  # the context's memory is released on exit
    else:
        r_np, c_np = extend_fn(T, Q, sd.cpu().numpy()[idx_np], params)
        rec = torch.from_numpy(np.ascontiguousarray(r_np).view(np.uint8).reshape(-1, REC_BYTES)).to(dev)
        cig = torch.frombuffer(bytearray(c_np), dtype=torch.uint8).to(dev) if c_np else \
            torch.zeros(0, dtype=torch.uint8, device=dev)
    t2 = time.perf_counter()
    # 3. gather to src and restore seed order
    pi = _gather_var(idx.view(torch.uint8), src, group)
    pr = _gather_var(rec.reshape(-1), src, group)
    pc = _gather_var(cig, src, group)
    out_rec = out_cig = None
    if rank == src:
        out, text = merge_shards([p.view(torch.int64) for p in pi], [p.view(-1, REC_BYTES) for p in pr], pc, n)
        if mark_redundant and mark_fn is None and out.is_cuda and n:
            fastz.fastz_mark_redundant_records_device(out, torch.cuda.current_device())
        out_rec = out.cpu().numpy().reshape(-1).view(fastz.ALIGN_DTYPE)
        out_cig = bytes(text.cpu().numpy().tobytes())
        if mark_redundant and mark_fn is not None:
            out_rec = np.ascontiguousarray(out_rec)
            mark_fn(out_rec)
        elif mark_redundant and not out.is_cuda:
            out_rec = np.ascontiguousarray(out_rec)
            fastz.fastz_mark_redundant_records(out_rec)
    t3 = time.perf_counter()
    if timings is not None:
        timings.update({"broadcast_s": t1 - t0, "extend_s": t2 - t1, "gather_s": t3 - t2})
    return out_rec, out_cig


def cuda_extend_fn(device: int):
    """An ``extend_fn`` running the CUDA path on host inputs (ASCII broadcast variant)."""
    def run(T: bytes, Q: bytes, seeds: np.ndarray, params):
        with fastz.Aligner(T, Q, params, device=device) as al:
            res = al.extend(seeds)
        return res.rec, res.cigar
    return run
