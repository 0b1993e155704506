"""The genome-pair driver over NCCL with the real CUDA path (world size 1: one GPU per box here)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

from paper_conf_sc_gundaboluvt21_b200 import dist as fzdist
from synth import genome
from tests.gpu_util import oparams

pytestmark = pytest.mark.gpu


def test_nccl_world1_matches_oracle():
    from oracle import core
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        w = genome.small_pair(31, length=20000, n_seeds=150)
        rec, cig = fzdist.extend_genome_pair(w.T, w.Q, w.seeds, mark_redundant=True)
    finally:
        dist.destroy_process_group()
    o = core.extend(w.T, w.Q, w.seeds, oparams())
    for f in ("score", "t_start", "t_end", "q_start", "q_end", "cigar_len"):
        assert np.array_equal(rec[f].astype(np.int64), o.rec[f]), f
    assert cig == o.cigar
    from oracle import dedup
    assert np.array_equal((rec["flags"] >> 5) & 1, dedup.redundant(o.rec))
