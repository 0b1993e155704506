"""Thin ctypes binding of libfastz.so (include/fastz.h).  Argument marshalling only: every step of the
hot path runs in the library's CUDA kernels.  There is no CPU fallback -- if libfastz.so is missing or no
CUDA device is present, the calls fail loudly.

Function names mirror the C ABI (fastz_create, fastz_extend_seeds, fastz_get_alignments, ...); the
:class:`Aligner` class wraps them for convenience.  PyTorch is used only to hand over device memory and
the current CUDA stream when the caller passes torch tensors.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# FASTZ_LIB: an alternative build of the same library (A/B experiments, tools/); default the in-tree build
LIB_PATH = os.environ.get("FASTZ_LIB") or os.path.join(HERE, "libfastz.so")

FASTZ_OK, FASTZ_EINVAL, FASTZ_EBASE, FASTZ_ERANGE = 0, -1, -2, -3
FASTZ_ENOMEM, FASTZ_ECUDA, FASTZ_ETRUNC, FASTZ_ESTATE = -4, -5, -6, -7
FLAG_ABOVE_K, FLAG_LEFT_EAGER, FLAG_RIGHT_EAGER, FLAG_OVERFLOW, FLAG_NO_CIGAR, FLAG_REDUNDANT = 1, 2, 4, 8, 16, 32
OPT_NO_EAGER, OPT_NO_TRIM, OPT_NO_BINNING, OPT_NO_BLOCK, OPT_TRACEBACK_ABOVE_K = 1, 2, 4, 8, 16
OPT_QUERY_REVCOMP = 32

# names declared in include/fastz.h (checked by tests/test_abi.py against the header)
EXPORTS = ["fastz_default_params", "fastz_create", "fastz_extend_seeds", "fastz_get_alignments",
           "fastz_get_alignments_device", "fastz_get_sides", "fastz_census", "fastz_get_stats",
           "fastz_destroy", "fastz_strerror", "fastz_int_peak", "fastz_default_seed_params", "fastz_find_hsps",
           "fastz_mark_redundant", "fastz_mark_redundant_records", "fastz_pack_sequence", "fastz_create_packed",
           "fastz_get_packed"]


class FastzError(RuntimeError):
    def __init__(self, status: int, text: str):
        super().__init__(f"fastz status {status}: {text}")
        self.status = status


class fastz_params(ctypes.Structure):
    _fields_ = [("sub", ctypes.c_int32 * 16), ("gap_open", ctypes.c_int32), ("gap_extend", ctypes.c_int32),
                ("ydrop", ctypes.c_int32), ("gapped_threshold", ctypes.c_int32), ("eager_max", ctypes.c_int32),
                ("options", ctypes.c_int32), ("n_score", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("dev_alloc", ctypes.c_void_p),
                ("dev_free", ctypes.c_void_p),
                ("alloc_user", ctypes.c_void_p)]


class fastz_stats(ctypes.Structure):
    _fields_ = [("ms_total", ctypes.c_float), ("ms_upload", ctypes.c_float), ("ms_inspect", ctypes.c_float),
                ("ms_bin", ctypes.c_float), ("ms_execute", ctypes.c_float), ("ms_traceback", ctypes.c_float),
                ("ms_combine", ctypes.c_float), ("n_warp_slots", ctypes.c_int32), ("n_seeds", ctypes.c_int64),
                ("n_sides", ctypes.c_int64), ("n_eager_sides", ctypes.c_int64), ("n_exec_sides", ctypes.c_int64),
                ("bin_counts", ctypes.c_int64 * 8), ("exec_words", ctypes.c_int64), ("cigar_bytes", ctypes.c_int64),
                ("n_launches", ctypes.c_int64), ("n_waves", ctypes.c_int64), ("n_escalated", ctypes.c_int64),
                ("n_wide_sides", ctypes.c_int64), ("exec_reserved_words", ctypes.c_int64),
                ("n_selfcheck_fail", ctypes.c_int64), ("n_packed_sides", ctypes.c_int64),
                ("n_long_sides", ctypes.c_int64), ("n_redo_sides", ctypes.c_int64)]


class fastz_seed_params(ctypes.Structure):
    _fields_ = [("pattern", ctypes.c_char * 64), ("transitions", ctypes.c_int32), ("xdrop", ctypes.c_int32),
                ("hspthresh", ctypes.c_int32), ("reserved", ctypes.c_int32)]


HSP_DTYPE = np.dtype([("t_start", "<i8"), ("q_start", "<i8"), ("length", "<i4"), ("score", "<i4")])
assert HSP_DTYPE.itemsize == 24

ALIGN_DTYPE = np.dtype([("score", "<i4"), ("left_score", "<i4"), ("right_score", "<i4"), ("flags", "<u4"),
                        ("t_start", "<i8"), ("t_end", "<i8"), ("q_start", "<i8"), ("q_end", "<i8"),
                        ("cigar_off", "<i8"), ("cigar_len", "<i4"), ("reserved", "<i4")])
assert ALIGN_DTYPE.itemsize == 64

_lib = None


def lib() -> ctypes.CDLL:
    """Load libfastz.so; raises if it has not been built (no fallback path exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_sc_gundaboluvt21_b200.build` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
    L.fastz_default_params.argtypes = [ctypes.POINTER(fastz_params)]
    L.fastz_default_params.restype = None
    L.fastz_create.argtypes = [ctypes.POINTER(fastz_params), vp, i64, vp, i64, i32, vp, ctypes.POINTER(vp)]
    L.fastz_extend_seeds.argtypes = [vp, vp, i64, i32]
    L.fastz_get_alignments.argtypes = [vp, vp, i64, vp, i64, ctypes.POINTER(i64), ctypes.POINTER(i64)]
    L.fastz_get_alignments_device.argtypes = [vp, ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(i64),
                                              ctypes.POINTER(i64)]
    L.fastz_get_sides.argtypes = [vp, vp, vp, vp, vp, i64]
    L.fastz_census.argtypes = [vp, vp, i64]
    L.fastz_mark_redundant.argtypes = [vp, vp, i64, ctypes.POINTER(i64)]
    L.fastz_mark_redundant_records.argtypes = [vp, i64, i32, vp, ctypes.POINTER(i64), i32]
    L.fastz_get_stats.argtypes = [vp, ctypes.POINTER(fastz_stats)]
    L.fastz_destroy.argtypes = [vp]
    L.fastz_destroy.restype = None
    L.fastz_strerror.argtypes = [i32]
    L.fastz_strerror.restype = ctypes.c_char_p
    L.fastz_int_peak.argtypes = [i32, ctypes.c_float, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]
    L.fastz_default_seed_params.argtypes = [ctypes.POINTER(fastz_seed_params)]
    L.fastz_default_seed_params.restype = None
    L.fastz_find_hsps.argtypes = [vp, ctypes.POINTER(fastz_seed_params), vp, vp, i64, ctypes.POINTER(i64),
                                  ctypes.POINTER(i64)]
    L.fastz_pack_sequence.argtypes = [vp, i64, i32, vp, vp, ctypes.POINTER(i32), i32, vp]
    L.fastz_create_packed.argtypes = [ctypes.POINTER(fastz_params), vp, vp, i64, vp, vp, i64, i32, vp,
                                      ctypes.POINTER(vp)]
    L.fastz_get_packed.argtypes = [vp, i32, ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(i64)]
    for name in ("fastz_pack_sequence", "fastz_create_packed", "fastz_get_packed", "fastz_mark_redundant",
                 "fastz_mark_redundant_records", "fastz_find_hsps", "fastz_create", "fastz_extend_seeds", "fastz_get_alignments", "fastz_get_alignments_device",
                 "fastz_get_sides", "fastz_census", "fastz_get_stats", "fastz_int_peak"):
        getattr(L, name).restype = i32
    _lib = L
    return L


def _check(status: int):
    if status != FASTZ_OK:
        raise FastzError(status, lib().fastz_strerror(status).decode())


# ----------------------------------------------------------------------------------- C-named wrappers

def fastz_default_params(**overrides) -> fastz_params:
    p = fastz_params()
    lib().fastz_default_params(ctypes.byref(p))
    for k, v in overrides.items():
        if k == "sub":
            flat = np.asarray(v, dtype=np.int32).reshape(16)
            for i in range(16):
                p.sub[i] = int(flat[i])
        else:
            setattr(p, k, int(v))
    return p


def _ptr_len(x):
    """(pointer, length, is_device) for bytes / numpy / torch inputs."""
    try:
        import torch
        if isinstance(x, torch.Tensor):
            x = x.contiguous()
            return x.data_ptr(), x.numel() * x.element_size(), x.is_cuda, x
    except ImportError:  # pragma: no cover
        pass
    if isinstance(x, str):
        x = x.encode()
    if isinstance(x, (bytes, bytearray)):
        arr = np.frombuffer(x, dtype=np.uint8)  # zero-copy view (the library only reads host inputs)
        return (arr.ctypes.data if len(x) else None), len(x), False, (arr, x)
    arr = np.ascontiguousarray(x)
    return arr.ctypes.data, arr.nbytes, False, arr


def fastz_create(params: fastz_params, target, query, device: int = 0, stream: int | None = None) -> int:
    tp, tl, _, tk = _ptr_len(target)
    qp, ql, _, qk = _ptr_len(query)
    out = ctypes.c_void_p()
    _check(lib().fastz_create(ctypes.byref(params), tp, tl, qp, ql, device, stream, ctypes.byref(out)))
    del tk, qk
    return out.value


def fastz_pack_sequence(seq, revcomp: bool = False, device: int = 0, stream: int | None = None):
    """ASCII (bytes / numpy / torch, host or device) -> (words int32 tensor, nmask int16 tensor, has_n) on
    cuda:device, as fastz_pack_sequence writes them (2-bit codes, 16 per word; 1-bit N mask)."""
    import torch
    sp, sl, _, keep = _ptr_len(seq)
    nw = (sl + 15) // 16
    dev = torch.device("cuda", device)
    words = torch.zeros(max(nw, 1), dtype=torch.int32, device=dev)
    nmask = torch.zeros(max(nw, 1), dtype=torch.int16, device=dev)
    has_n = ctypes.c_int32()
    _check(lib().fastz_pack_sequence(sp, sl, 1 if revcomp else 0, words.data_ptr(), nmask.data_ptr(),
                                     ctypes.byref(has_n), device, stream))
    del keep
    return words[:nw], nmask[:nw], bool(has_n.value)


def fastz_create_packed(params: fastz_params, t_words, t_nmask, tlen: int, q_words, q_nmask, qlen: int,
                        device: int = 0, stream: int | None = None) -> int:
    """Context from packed device tensors (``fastz_pack_sequence`` layout); a mask may be None (no N)."""
    out = ctypes.c_void_p()
    ptr = lambda t: None if t is None else t.data_ptr()  # noqa: E731
    _check(lib().fastz_create_packed(ctypes.byref(params), ptr(t_words), ptr(t_nmask), int(tlen), ptr(q_words),
                                     ptr(q_nmask), int(qlen), device, stream, ctypes.byref(out)))
    return out.value


def fastz_extend_seeds(ctx: int, seeds) -> int:
    """seeds: (n, 2) int64 cut points as numpy (host) or a CUDA torch tensor (device)."""
    try:
        import torch
        if isinstance(seeds, torch.Tensor):
            s = seeds.to(torch.int64).contiguous()
            _check(lib().fastz_extend_seeds(ctx, s.data_ptr(), s.shape[0], 1 if s.is_cuda else 0))
            return s.shape[0]
    except ImportError:  # pragma: no cover
        pass
    s = np.ascontiguousarray(np.asarray(seeds, dtype=np.int64).reshape(-1, 2))
    _check(lib().fastz_extend_seeds(ctx, s.ctypes.data, s.shape[0], 0))
    return s.shape[0]


def fastz_get_alignments(ctx: int):
    n, nb = ctypes.c_int64(), ctypes.c_int64()
    st = lib().fastz_get_alignments(ctx, None, 0, None, 0, ctypes.byref(n), ctypes.byref(nb))
    if st not in (FASTZ_OK, FASTZ_ETRUNC):
        _check(st)
    rec = np.empty(max(n.value, 1), dtype=ALIGN_DTYPE)
    cig = ctypes.create_string_buffer(max(nb.value, 1))
    _check(lib().fastz_get_alignments(ctx, rec.ctypes.data, n.value, cig, nb.value, ctypes.byref(n), ctypes.byref(nb)))
    return rec[:n.value], cig.raw[:nb.value]


class _DevView:
    """__cuda_array_interface__ over library-owned device memory (zero-copy torch.as_tensor)."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr or 0, False),
                                         "version": 3, "strides": None}


def fastz_get_alignments_device(ctx: int, device: int = 0):
    """(records uint8[n, 64], cigar uint8[bytes]) as torch tensors ALIASING the context's device memory (valid
    until the next extend / destroy).  The caller must order its reads after the context's stream."""
    import torch
    recs, cig = ctypes.c_void_p(), ctypes.c_void_p()
    n, nb = ctypes.c_int64(), ctypes.c_int64()
    _check(lib().fastz_get_alignments_device(ctx, ctypes.byref(recs), ctypes.byref(cig), ctypes.byref(n),
                                             ctypes.byref(nb)))
    dev = torch.device("cuda", device)
    r = torch.as_tensor(_DevView(recs.value, n.value * 64), device=dev).view(n.value, 64) if n.value else \
        torch.zeros((0, 64), dtype=torch.uint8, device=dev)
    c = torch.as_tensor(_DevView(cig.value, nb.value), device=dev) if nb.value else \
        torch.zeros(0, dtype=torch.uint8, device=dev)
    return r, c


def fastz_get_sides(ctx: int, n: int):
    score = np.zeros(max(2 * n, 1), np.int32)
    ti = np.zeros_like(score)
    qj = np.zeros_like(score)
    fl = np.zeros(max(2 * n, 1), np.uint32)
    _check(lib().fastz_get_sides(ctx, score.ctypes.data, ti.ctypes.data, qj.ctypes.data, fl.ctypes.data, 2 * n))
    return score[:2 * n], ti[:2 * n], qj[:2 * n], fl[:2 * n]


def fastz_census(ctx: int, n: int) -> np.ndarray:
    cells = np.zeros(max(2 * n, 1), np.int64)
    _check(lib().fastz_census(ctx, cells.ctypes.data, 2 * n))
    return cells[:2 * n]


def fastz_mark_redundant(ctx: int, n: int):
    """Redundant-alignment post-pass (NEXT-3, reading R14) on the last batch: returns (uint8[n] marks, count)."""
    red = np.zeros(max(n, 1), np.uint8)
    cnt = ctypes.c_int64()
    _check(lib().fastz_mark_redundant(ctx, red.ctypes.data, n, ctypes.byref(cnt)))
    return red[:n], cnt.value


def fastz_mark_redundant_records(rec: np.ndarray, device: int = 0):
    """Context-free post-pass (reading R14) on a host ALIGN_DTYPE array: sets FLAG_REDUNDANT in rec["flags"] in
    place (the array must be C-contiguous) and returns (uint8[n] marks, count)."""
    if rec.dtype != ALIGN_DTYPE or not rec.flags["C_CONTIGUOUS"] or not rec.flags["WRITEABLE"]:
        raise ValueError("rec must be a writeable C-contiguous ALIGN_DTYPE array")
    n = len(rec)
    red = np.zeros(max(n, 1), np.uint8)
    cnt = ctypes.c_int64()
    _check(lib().fastz_mark_redundant_records(rec.ctypes.data if n else None, n, 0, red.ctypes.data,
                                              ctypes.byref(cnt), device))
    return red[:n], cnt.value


def fastz_mark_redundant_records_device(rec, device: int = 0) -> int:
    """Context-free post-pass (reading R14) on DEVICE records (a contiguous CUDA tensor holding n x 64-byte
    fastz_alignment records): sets FLAG_REDUNDANT in place; returns the count.  Orders itself after the
    current PyTorch stream."""
    import torch
    n = rec.numel() // ALIGN_DTYPE.itemsize
    torch.cuda.current_stream(rec.device).synchronize()
    cnt = ctypes.c_int64()
    _check(lib().fastz_mark_redundant_records(rec.data_ptr() if n else None, n, 1, None, ctypes.byref(cnt), device))
    return cnt.value


def fastz_get_stats(ctx: int) -> dict:
    s = fastz_stats()
    _check(lib().fastz_get_stats(ctx, ctypes.byref(s)))
    d = {k: getattr(s, k) for k, _ in fastz_stats._fields_}
    d["bin_counts"] = list(s.bin_counts)
    return d


def fastz_destroy(ctx: int):
    if ctx:
        lib().fastz_destroy(ctx)


def fastz_default_seed_params(**overrides) -> fastz_seed_params:
    sp = fastz_seed_params()
    lib().fastz_default_seed_params(ctypes.byref(sp))
    for k, v in overrides.items():
        setattr(sp, k, v.encode() if k == "pattern" else int(v))
    return sp


def fastz_find_hsps(ctx: int, sp: fastz_seed_params | None = None):
    """(HSPs as a HSP_DTYPE array in anchor order, anchors as an (n, 2) int64 array, raw hit count)."""
    sp = sp if sp is not None else fastz_default_seed_params()
    n, hits = ctypes.c_int64(0), ctypes.c_int64(0)
    st = lib().fastz_find_hsps(ctx, ctypes.byref(sp), None, None, 0, ctypes.byref(n), ctypes.byref(hits))
    if st not in (FASTZ_OK, FASTZ_ETRUNC):
        _check(st)
    cap = int(n.value)
    hs = np.zeros(cap, dtype=HSP_DTYPE)
    an = np.zeros((cap, 2), dtype=np.int64)
    if cap:
        _check(lib().fastz_find_hsps(ctx, ctypes.byref(sp), hs.ctypes.data, an.ctypes.data, cap, ctypes.byref(n),
                                     ctypes.byref(hits)))
    return hs, an, int(hits.value)


def fastz_int_peak(device: int = 0, ms: float = 200.0):
    ops, mhz = ctypes.c_double(), ctypes.c_double()
    _check(lib().fastz_int_peak(device, ms, ctypes.byref(ops), ctypes.byref(mhz)))
    return ops.value, mhz.value


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)


def torch_allocator_hooks(device: int = 0):
    """(dev_alloc, dev_free) C callbacks that route the context's device memory through PyTorch's caching
    allocator (on the context's stream), so freed pools are reused by later contexts without cudaMalloc/cudaFree.
    Keep the returned objects alive as long as the context."""
    import torch

    def _alloc(nbytes, stream, user):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), device, stream or 0)
        except Exception:  # out of memory: the library reports FASTZ_ENOMEM
            return None

    def _free(ptr, stream, user):
        if ptr:
            torch.cuda.caching_allocator_delete(ptr)

    return _ALLOC_FN(_alloc), _FREE_FN(_free)


# ----------------------------------------------------------------------------------- convenience class

@dataclass
class PackedSequence:
    """A 2-bit packed sequence on the device (``fastz_pack_sequence`` layout); nmask None = no N."""
    words: object
    nmask: object
    length: int

    @staticmethod
    def pack(seq, revcomp: bool = False, device: int = 0, stream: int | None = None) -> "PackedSequence":
        w, m, has_n = fastz_pack_sequence(seq, revcomp, device, stream)
        n = len(seq) if not hasattr(seq, "numel") else seq.numel()
        return PackedSequence(w, m if has_n else None, int(n))


@dataclass
class Alignments:
    rec: np.ndarray
    cigar: bytes = field(repr=False)

    def cigar_of(self, s: int) -> str:
        r = self.rec[s]
        c = self.cigar[r["cigar_off"]: r["cigar_off"] + r["cigar_len"]]
        return (c.tobytes() if isinstance(c, np.ndarray) else c).decode()


class Aligner:
    """One context (device + stream + packed sequences).  ``extend`` returns host results; ``extend_only``
    leaves them on the device (for timing / NCCL gathers)."""

    def __init__(self, target, query, params: fastz_params | None = None, device: int = 0, stream=None,
                 torch_alloc: bool = False, **kw):
        self.params = params if params is not None else fastz_default_params(**kw)
        if torch_alloc:  # device memory through PyTorch's caching allocator (fastz_params.dev_alloc / dev_free)
            self._hooks = torch_allocator_hooks(device)
            self.params.dev_alloc = ctypes.cast(self._hooks[0], ctypes.c_void_p)
            self.params.dev_free = ctypes.cast(self._hooks[1], ctypes.c_void_p)
        if stream is None:
            try:
                import torch
                if torch.cuda.is_available():
                    torch.cuda.set_device(device)
                    stream = torch.cuda.current_stream(device).cuda_stream
            except ImportError:  # pragma: no cover
                stream = None
        self.device = device
        self.stream = stream
        if isinstance(target, PackedSequence):
            self.ctx = fastz_create_packed(self.params, target.words, target.nmask, target.length, query.words,
                                           query.nmask, query.length, device, stream)
        else:
            self.ctx = fastz_create(self.params, target, query, device, stream)
        self.n = 0

    def extend_only(self, seeds) -> int:
        try:
            import torch
            if isinstance(seeds, torch.Tensor) and seeds.is_cuda:
                seeds = seeds.to(torch.int64).contiguous()
                cur = torch.cuda.current_stream(seeds.device)
                if cur.cuda_stream != (self.stream or 0):
                    cur.synchronize()  # the seeds were produced on another stream than the context's
        except ImportError:  # pragma: no cover
            pass
        self.n = fastz_extend_seeds(self.ctx, seeds)
        return self.n

    def extend(self, seeds) -> Alignments:
        self.extend_only(seeds)
        rec, cig = fastz_get_alignments(self.ctx)
        return Alignments(rec, cig)

    def results_device(self):
        """(records uint8[n, 64], cigar uint8[bytes]) torch tensors aliasing the context's device memory, with the
        context's stream synchronized (so any stream may read them)."""
        import torch
        r, c = fastz_get_alignments_device(self.ctx, self.device)
        if self.stream:
            torch.cuda.ExternalStream(self.stream, device=torch.device("cuda", self.device)).synchronize()
        else:
            torch.cuda.synchronize(self.device)
        return r, c

    def results(self) -> Alignments:
        rec, cig = fastz_get_alignments(self.ctx)
        return Alignments(rec, cig)

    def results_pinned(self) -> Alignments:
        """Like ``results`` but copies into page-locked host buffers owned by this Aligner and reused by the
        next call (DMA-speed copies, no page faults); the returned arrays are views valid until then."""
        import torch
        n, nb = ctypes.c_int64(), ctypes.c_int64()
        st = lib().fastz_get_alignments(self.ctx, None, 0, None, 0, ctypes.byref(n), ctypes.byref(nb))
        if st not in (FASTZ_OK, FASTZ_ETRUNC):
            _check(st)
        need_r, need_c = max(n.value, 1) * ALIGN_DTYPE.itemsize, max(nb.value, 1)
        if getattr(self, "_pin_rec", None) is None or self._pin_rec.numel() < need_r:
            self._pin_rec = torch.empty(need_r + need_r // 4, dtype=torch.uint8, pin_memory=True)
        if getattr(self, "_pin_cig", None) is None or self._pin_cig.numel() < need_c:
            self._pin_cig = torch.empty(need_c + need_c // 4, dtype=torch.uint8, pin_memory=True)
        _check(lib().fastz_get_alignments(self.ctx, self._pin_rec.data_ptr(), n.value, self._pin_cig.data_ptr(),
                                          nb.value, ctypes.byref(n), ctypes.byref(nb)))
        rec = self._pin_rec.numpy()[: n.value * ALIGN_DTYPE.itemsize].view(ALIGN_DTYPE)
        return Alignments(rec, self._pin_cig.numpy()[: nb.value])

    def sides(self):
        return fastz_get_sides(self.ctx, self.n)

    def find_hsps(self, **seed_params):
        """Seeding + ungapped filter on this context's sequences (NEXT-4): (hsps, anchors, hits)."""
        return fastz_find_hsps(self.ctx, fastz_default_seed_params(**seed_params))

    def mark_redundant(self):
        """fastz_mark_redundant on the last batch: (uint8[n] marks, count); sets FLAG_REDUNDANT in the records."""
        return fastz_mark_redundant(self.ctx, self.n)

    def census(self) -> np.ndarray:
        return fastz_census(self.ctx, self.n)

    def stats(self) -> dict:
        return fastz_get_stats(self.ctx)

    def close(self):
        fastz_destroy(self.ctx)
        self.ctx = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            if self.ctx:
                self.close()
        except Exception:
            pass
