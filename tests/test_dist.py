"""Multi-process tests of the genome-pair driver (paper_conf_sc_gundaboluvt21_b200.dist) with the gloo
backend at world size 2 on CPU.  The per-rank compute is injected (the CPU oracle here, test
infrastructure); the sharding, broadcast, gather and seed-order reassembly are the product code."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_gundaboluvt21_b200 import dist as fzdist


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_fn(T, Q, seeds, params):
    from oracle import core
    from paper_conf_sc_gundaboluvt21_b200.fastz import ALIGN_DTYPE
    r = core.extend(T, Q, seeds, threads=2)
    out = np.zeros(len(seeds), dtype=ALIGN_DTYPE)
    for f in ("score", "left_score", "right_score", "t_start", "t_end", "q_start", "q_end", "cigar_off", "cigar_len"):
        out[f] = r.rec[f]
    out["flags"] = r.rec["flags"]
    return out, r.cigar


def _oracle_mark(rec):
    from oracle import dedup
    rec["flags"] |= dedup.redundant(rec).astype(np.uint32) << 5   # FLAG_REDUNDANT = 32


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from synth import genome
        w = genome.small_pair(21, length=8000, n_seeds=90)
        rec, cig = fzdist.extend_genome_pair(w.T if rank == 0 else None, w.Q if rank == 0 else None,
                                             w.seeds if rank == 0 else None, extend_fn=_oracle_fn,
                                             mark_redundant=True, mark_fn=_oracle_mark)
        if rank == 0:
            q.put((rec.tobytes(), cig))
    finally:
        dist.destroy_process_group()


def test_shard_indices_partition():
    for n in (0, 1, 7, 1000):
        for world in (1, 2, 3, 8):
            parts = [fzdist.shard_indices(n, world, r) for r in range(world)]
            allp = np.concatenate(parts) if parts else np.zeros(0)
            assert sorted(allp.tolist()) == list(range(n))
            assert max(len(p) for p in parts) - min(len(p) for p in parts) <= 1


@pytest.mark.parametrize("world", [2])
def test_gloo_world2_matches_single_process(world):
    from synth import genome
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    rec_bytes, cig = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    w = genome.small_pair(21, length=8000, n_seeds=90)
    ref_rec, ref_cig = _oracle_fn(w.T, w.Q, w.seeds, None)
    # the post-pass runs once over the gathered WHOLE set (marks depend on every record, not one shard's)
    _oracle_mark(ref_rec)
    assert (ref_rec["flags"] & 32).any()
    assert rec_bytes == ref_rec.tobytes() and cig == ref_cig
