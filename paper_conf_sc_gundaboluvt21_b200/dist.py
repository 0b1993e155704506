"""Multi-GPU genome-pair driver (one process per GPU, torch.distributed over NCCL / NVLink).

Seed extensions are independent ("the seeds can be partitioned easily"), so the only
collectives are at the edges of the path:

1. rank 0 broadcasts the two ASCII sequences (each rank packs them on its own GPU inside ``fastz_create``);
2. seeds are permuted by a fixed hash and cut into W contiguous shards (spreads the unknown-length long tail);
3. every rank runs the CUDA path on its shard (no communication);
4. per-rank record counts / CIGAR sizes are all-gathered, then records (64 B each) and CIGAR bytes are gathered
   to rank 0 and put back in seed order.

Results are byte-identical for any world size.  ``extend_fn`` is injectable so the host-side plumbing can be
tested with the gloo backend on CPU; the default is the CUDA path (``fastz.Aligner``).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import fastz

_HASH = np.uint64(0x9E3779B97F4A7C15)


def shard_order(n: int) -> np.ndarray:
    """Deterministic pseudo-random permutation of seed indices (multiplicative hash, stable argsort)."""
    h = (np.arange(n, dtype=np.uint64) * _HASH) ^ np.uint64(0xD1B54A32D192ED03)
    h ^= h >> np.uint64(29)
    return np.argsort(h, kind="stable").astype(np.int64)


def shard_indices(n: int, world: int, rank: int) -> np.ndarray:
    order = shard_order(n)
    lo = (n * rank) // world
    hi = (n * (rank + 1)) // world
    return np.sort(order[lo:hi])


def _dev(group=None) -> torch.device:
    if dist.get_backend(group) == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def broadcast_bytes(data: bytes | None, src: int = 0, group=None) -> bytes:
    dev = _dev(group)
    rank = dist.get_rank(group)
    n = torch.tensor([len(data) if rank == src else 0], dtype=torch.int64, device=dev)
    dist.broadcast(n, src, group=group)
    if rank == src:
        buf = torch.frombuffer(bytearray(data), dtype=torch.uint8).to(dev) if len(data) else \
            torch.zeros(0, dtype=torch.uint8, device=dev)
    else:
        buf = torch.empty(int(n.item()), dtype=torch.uint8, device=dev)
    if int(n.item()):
        dist.broadcast(buf, src, group=group)
    return bytes(buf.cpu().numpy().tobytes())


def broadcast_array(a: np.ndarray | None, src: int = 0, group=None, dtype=np.int64) -> np.ndarray:
    raw = broadcast_bytes(a.astype(dtype).tobytes() if a is not None else None, src, group)
    return np.frombuffer(raw, dtype=dtype).copy()


def _gather_var(payload: np.ndarray, group=None, dst: int = 0):
    """Gather variable-length uint8 payloads to ``dst`` (all_gather of sizes, padded gather)."""
    dev = _dev(group)
    world = dist.get_world_size(group)
    sz = torch.tensor([payload.nbytes], dtype=torch.int64, device=dev)
    sizes = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(sizes, sz, group=group)
    sizes = [int(s.item()) for s in sizes]
    mx = max(max(sizes), 1)
    buf = torch.zeros(mx, dtype=torch.uint8, device=dev)
    if payload.nbytes:
        buf[:payload.nbytes] = torch.from_numpy(payload.view(np.uint8).copy()).to(dev)
    if dist.get_rank(group) == dst:
        bufs = [torch.zeros(mx, dtype=torch.uint8, device=dev) for _ in range(world)]
        dist.gather(buf, bufs, dst=dst, group=group)
        return [bufs[r][:sizes[r]].cpu().numpy() for r in range(world)]
    dist.gather(buf, None, dst=dst, group=group)
    return None


def gather_results(idx: np.ndarray, rec: np.ndarray, cigar: bytes, n: int, group=None, dst: int = 0):
    """Gather per-rank (seed indices, records, CIGAR text) to ``dst`` and restore seed order."""
    parts_idx = _gather_var(idx.astype(np.int64), group, dst)
    parts_rec = _gather_var(np.ascontiguousarray(rec), group, dst)
    parts_cig = _gather_var(np.frombuffer(cigar, dtype=np.uint8) if cigar else np.zeros(0, np.uint8), group, dst)
    if dist.get_rank(group) != dst:
        return None, None
    out = np.zeros(n, dtype=rec.dtype)
    texts = [None] * n
    for pi, pr, pc in zip(parts_idx, parts_rec, parts_cig):
        ii = pi.view(np.int64)
        rr = pr.view(rec.dtype)
        cc = pc.tobytes()
        for k, s in enumerate(ii):
            r = rr[k]
            texts[s] = cc[r["cigar_off"]: r["cigar_off"] + r["cigar_len"]]
            out[s] = r
    off = 0
    for s in range(n):
        out[s]["cigar_off"] = off
        off += len(texts[s])
    return out, b"".join(texts)


def cuda_extend_fn(device: int):
    def run(T: bytes, Q: bytes, seeds: np.ndarray, params):
        with fastz.Aligner(T, Q, params, device=device) as al:
            res = al.extend(seeds)
        return res.rec, res.cigar
    return run


def extend_genome_pair(T: bytes | None, Q: bytes | None, seeds: np.ndarray | None, params=None, group=None,
                       extend_fn=None, src: int = 0, mark_redundant: bool = False, mark_fn=None):
    """Collective: every rank calls it; only ``src`` needs real inputs.  Returns (records, cigar) on ``src``
    (seed order), (None, None) elsewhere.  ``mark_redundant``: after the gather, ``src`` runs the
    redundant-alignment post-pass (NEXT-3, reading R14) over the WHOLE record set -- the marks depend on every
    record, so they cannot be taken per shard -- setting FLAG_REDUNDANT in place (``mark_fn(rec)``, default the
    CUDA ``fastz_mark_redundant_records`` on the current device)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    T = broadcast_bytes(T, src, group)
    Q = broadcast_bytes(Q, src, group)
    seeds = broadcast_array(None if seeds is None else np.asarray(seeds, np.int64).reshape(-1), src, group)
    seeds = seeds.reshape(-1, 2)
    n = len(seeds)
    idx = shard_indices(n, world, rank)
    if extend_fn is None:
        extend_fn = cuda_extend_fn(torch.cuda.current_device())
    rec, cig = extend_fn(T, Q, seeds[idx], params)
    out_rec, out_cig = gather_results(idx, rec, cig, n, group, src)
    if mark_redundant and out_rec is not None:
        out_rec = np.ascontiguousarray(out_rec)
        if mark_fn is None:
            fastz.fastz_mark_redundant_records(out_rec, torch.cuda.current_device())
        else:
            mark_fn(out_rec)
    return out_rec, out_cig
