"""C-ABI behaviour on the GPU: input forms (host/device, lowercase), error codes and buffer protocols."""
import ctypes

import numpy as np
import pytest
import torch

from paper_conf_sc_gundaboluvt21_b200 import fastz
from synth import genome

pytestmark = pytest.mark.gpu


def _w():
    return genome.small_pair(80, length=12000, n_seeds=100)


def test_lowercase_equals_uppercase():
    w = _w()
    with fastz.Aligner(w.T, w.Q) as a, fastz.Aligner(w.T.lower(), w.Q.lower()) as b:
        ra, rb = a.extend(w.seeds), b.extend(w.seeds)
    assert np.array_equal(ra.rec, rb.rec) and ra.cigar == rb.cigar


def test_device_sequences_and_device_seeds_equal_host():
    w = _w()
    T = torch.frombuffer(bytearray(w.T), dtype=torch.uint8).cuda()
    Q = torch.frombuffer(bytearray(w.Q), dtype=torch.uint8).cuda()
    with fastz.Aligner(w.T, w.Q) as a, fastz.Aligner(T, Q) as b:
        ra = a.extend(w.seeds)
        rb = b.extend(torch.from_numpy(w.seeds).cuda())
    assert np.array_equal(ra.rec, rb.rec) and ra.cigar == rb.cigar


def test_invalid_base_reports_index():
    with pytest.raises(fastz.FastzError) as e:
        fastz.Aligner(b"ACGTXACGT", b"ACGT")
    assert e.value.status == fastz.FASTZ_EBASE and "index 4" in str(e.value)
    with pytest.raises(fastz.FastzError) as e:
        fastz.Aligner(b"ACGT", b"AC-T")
    assert e.value.status == fastz.FASTZ_EBASE


def test_seed_out_of_range():
    with fastz.Aligner(b"ACGTACGT", b"ACGTACGT") as a:
        with pytest.raises(fastz.FastzError) as e:
            a.extend(np.array([[1, 1], [9, 2]], np.int64))
        assert e.value.status == fastz.FASTZ_ERANGE and "seed 1" in str(e.value)
        with pytest.raises(fastz.FastzError):
            a.extend(np.array([[-1, 0]], np.int64))


def test_estate_and_etrunc():
    L = fastz.lib()
    w = _w()
    ctx = fastz.fastz_create(fastz.fastz_default_params(), w.T, w.Q, 0)
    try:
        n, nb = ctypes.c_int64(), ctypes.c_int64()
        assert L.fastz_get_alignments(ctx, None, 0, None, 0, ctypes.byref(n), ctypes.byref(nb)) == fastz.FASTZ_ESTATE
        fastz.fastz_extend_seeds(ctx, w.seeds)
        rc = L.fastz_get_alignments(ctx, None, 0, None, 0, ctypes.byref(n), ctypes.byref(nb))
        assert rc == fastz.FASTZ_ETRUNC and n.value == len(w.seeds) and nb.value > 0
        rec = np.zeros(n.value, dtype=fastz.ALIGN_DTYPE)
        small = ctypes.create_string_buffer(nb.value - 1)
        rc = L.fastz_get_alignments(ctx, rec.ctypes.data, n.value, small, nb.value - 1, ctypes.byref(n), ctypes.byref(nb))
        assert rc == fastz.FASTZ_ETRUNC
        full = ctypes.create_string_buffer(nb.value)
        assert L.fastz_get_alignments(ctx, rec.ctypes.data, n.value, full, nb.value, ctypes.byref(n),
                                      ctypes.byref(nb)) == 0
        recs, cig = ctypes.c_void_p(), ctypes.c_void_p()
        assert L.fastz_get_alignments_device(ctx, ctypes.byref(recs), ctypes.byref(cig), ctypes.byref(n),
                                             ctypes.byref(nb)) == 0
        assert recs.value and cig.value
    finally:
        fastz.fastz_destroy(ctx)


def test_repeated_batches_reuse_context():
    w = _w()
    with fastz.Aligner(w.T, w.Q) as a:
        r1 = a.extend(w.seeds)
        r2 = a.extend(w.seeds[:10])
        r3 = a.extend(w.seeds)
    assert np.array_equal(r1.rec, r3.rec) and r1.cigar == r3.cigar
    assert np.array_equal(r2.rec[:10]["score"], r1.rec[:10]["score"])


def test_int_peak_is_sane():
    ops, mhz = fastz.fastz_int_peak(0, 50.0)
    assert 1e12 < ops < 1e14 and 500 < mhz < 3000


def test_results_pinned_equal_results():
    """Page-locked reusable output buffers (the e2e path of bench.py) give the same records and CIGARs."""
    w = _w()
    with fastz.Aligner(w.T, w.Q) as a:
        r = a.extend(w.seeds)
        p = a.results_pinned()
        assert np.array_equal(r.rec, p.rec) and r.cigar == p.cigar.tobytes()
        assert all(r.cigar_of(s) == p.cigar_of(s) for s in range(0, len(w.seeds), 7))
        a.extend(w.seeds[:10])           # smaller batch: buffers reused, views shrink
        p2 = a.results_pinned()
        assert len(p2.rec) == 10
        assert all(p2.cigar_of(s) == r.cigar_of(s) for s in range(10))


def test_torch_caching_allocator_hooks():
    """fastz_params.dev_alloc / dev_free routed through PyTorch's caching allocator: identical results, and the
    context's blocks return to PyTorch's cache on destroy (reused by the next context)."""
    w = _w()
    with fastz.Aligner(w.T, w.Q) as a:
        ra = a.extend(w.seeds)
    before = torch.cuda.memory_allocated()
    with fastz.Aligner(w.T, w.Q, torch_alloc=True) as b:
        rb = b.extend(w.seeds)
        assert torch.cuda.memory_allocated() > before      # the context's buffers live in PyTorch's pool
        hs, an, _ = b.find_hsps(hspthresh=500)
    assert np.array_equal(ra.rec, rb.rec) and ra.cigar == rb.cigar
    assert torch.cuda.memory_allocated() == before         # all returned on destroy
    with fastz.Aligner(w.T, w.Q, torch_alloc=True) as c:   # reuses the cached blocks
        rc = c.extend(w.seeds)
    assert np.array_equal(ra.rec, rc.rec)


def test_packed_contexts_equal_ascii_contexts():
    """fastz_pack_sequence + fastz_create_packed (the multi-GPU broadcast format) give the same results as
    fastz_create from ASCII: plain, with N bases (masks), and the minus strand (revcomp packing)."""
    w = _w()
    T = bytearray(w.T)
    T[100:130] = b"N" * 30
    T = bytes(T)
    for tq, opts in (((w.T, w.Q), 0), ((T, w.Q.lower()), 0), ((w.T, w.Q), fastz.OPT_QUERY_REVCOMP)):
        with fastz.Aligner(tq[0], tq[1], fastz.fastz_default_params(options=opts)) as a:
            ra = a.extend(w.seeds)
        pt = fastz.PackedSequence.pack(tq[0])
        pq = fastz.PackedSequence.pack(tq[1], revcomp=bool(opts & fastz.OPT_QUERY_REVCOMP))
        assert (pt.nmask is not None) == (b"N" in tq[0])
        with fastz.Aligner(pt, pq) as b:
            rb = b.extend(w.seeds)
            rd, cd = b.results_device()
            assert rd.shape == (len(w.seeds), 64) and cd.numel() == len(rb.cigar)
            assert rd.cpu().numpy().tobytes() == rb.rec.tobytes() and cd.cpu().numpy().tobytes() == rb.cigar
        assert np.array_equal(ra.rec, rb.rec) and ra.cigar == rb.cigar


def test_pack_sequence_rejects_invalid_base():
    with pytest.raises(fastz.FastzError) as e:
        fastz.fastz_pack_sequence(b"ACGTACGTACGTACGTACGX")
    assert e.value.status == fastz.FASTZ_EBASE and "index 19" in str(e.value)
