// api.cu -- host side of libfastz.so: the C ABI of include/fastz.h.
//
// Pipeline of fastz_extend_seeds (one stream, two host syncs):
//   seeds H2D -> validate -> inspector (persistent warps, eager traceback inside) -> binning + exclusive
//   scans of the executor sizes (static allocation from inspector sizes) -> [sync: D2H of 8 totals,
//   grow the traceback pool] -> executor (trimmed, larger bins first) -> traceback -> CIGAR length pass +
//   scan -> [sync: CIGAR bytes] -> CIGAR/record write.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../../include/fastz.h"
#include "internal.h"

using namespace fz;

namespace {

thread_local std::string g_err;

int fail(int code, const std::string& msg) {
    g_err = msg;
    return code;
}

#define CK(x)                                                                                  \
    do {                                                                                       \
        cudaError_t _e = (x);                                                                  \
        if (_e != cudaSuccess)                                                                 \
            return fail(_e == cudaErrorMemoryAllocation ? FASTZ_ENOMEM : FASTZ_ECUDA,          \
                        std::string(#x) + ": " + cudaGetErrorString(_e));                       \
    } while (0)

// NVTX range for external profilers (Nsight Systems / Compute): host-side stage markers of fastz_extend_seeds
// (enqueue + the two host syncs); header-only NVTX v3, a no-op without a profiler attached
struct Nvtx {
    bool on = true;
    explicit Nvtx(const char* name) { nvtxRangePushA(name); }
    void end() {
        if (on) nvtxRangePop();
        on = false;
    }
    ~Nvtx() { end(); }
    Nvtx(const Nvtx&) = delete;
    Nvtx& operator=(const Nvtx&) = delete;
};

struct DBuf {
    void* p = nullptr;
    size_t cap = 0;
};

}  // namespace

struct fastz_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    fastz_params prm{};
    DevParams dp{};
    int tlen = 0, qlen = 0;
    DBuf Tf, Tr, Qf, Qr, stage;
    DBuf TfN, TrN, QfN, QrN;  // N masks (1 bit per base, 16 per u16 word)
    bool t_has_n = false, q_has_n = false;
    DBuf seeds, score, ti, qj, flags, eops, bound, maxsw, esc, nstrip;
    DBuf woff, soff, roff, bin, list, counters, totals, tmpa, tmpb, tmpc, scan_tmp, wl, wlo;
    DBuf codes, stab, runs, nruns, ciglen, cigar, recs, cells, ring, small, wide, ring2, lpt_tmp, order_tmp, order_buf;
    DBuf ring_pair, redo;  // packed inspector (pair.cuh): two rings of int2 per warp slot; abandoned sides
    DBuf pdbg;             // FASTZ_PAIR_DEBUG diagnostics
    DBuf phist;            // packed inspector: per warp slot and half, strip history (exact executor reservation)
    // seeding (fastz_find_hsps)
    DBuf s_kin, s_kout, s_pin, s_pout, s_start, s_cnt, s_off, s_hits, s_hsp, s_keep, s_sel, s_list, s_list2,
        s_k1, s_k2, s_i1, s_i2, s_flag, s_pos, s_out, s_anch, s_tmp;
    // redundant-alignment post-pass (fastz_mark_redundant)
    DBuf r_k1, r_k2, r_i1, r_i2, r_box, r_sc, r_red, r_tmp, r_cnt;
    int R = 4, grid = 0, nslots = 0, rmask = 0;
    // packed inspector: launch grid (0 = not built for this context), constants, whether the parameters admit it
    int grid_mixed = 0;
    PairParams pq{};
    bool pair_params_ok = false;
    int64_t n_pair_sides = 0, n_redo_sides = 0, n_long_sides = 0;
    // wide ring of the last batch (sides whose explored band overflowed `ring`): grid2 CTAs x WARPS slots of
    // rmask2 + 1 entries; nwide sides listed in `wide`
    int grid2 = 0, rmask2 = 0, nwide = 0;
    int64_t n = 0, cigar_bytes = 0, nexec = 0;
    int nwaves = 0;
    bool have = false;
    fastz_stats stats{};
    cudaEvent_t ev[8] = {};
    // second stream: the 32-bit inspector of the predicted-long sides runs beside the packed inspector
    cudaStream_t side_stream = nullptr;
    cudaEvent_t fork_ev = nullptr, join_ev = nullptr;
    bool ev_ok = false;
};

namespace {

int dalloc(fastz_ctx* c, DBuf& b, size_t bytes) {
    if (bytes <= b.cap && b.p) return 0;
    size_t want = std::max<size_t>(bytes + bytes / 4, 256);
    if (b.p) {
        cudaStreamSynchronize(c->stream);
        if (c->prm.dev_free) c->prm.dev_free(b.p, c->stream, c->prm.alloc_user);
        else cudaFree(b.p);
        b.p = nullptr;
        b.cap = 0;
    }
    void* p = nullptr;
    if (c->prm.dev_alloc) {
        p = c->prm.dev_alloc(want, c->stream, c->prm.alloc_user);
        if (!p) return fail(FASTZ_ENOMEM, "dev_alloc hook returned NULL for " + std::to_string(want) + " bytes");
    } else {
        cudaError_t e = cudaMalloc(&p, want);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(FASTZ_ENOMEM, "cudaMalloc(" + std::to_string(want) + "): " + cudaGetErrorString(e));
        }
    }
    b.p = p;
    b.cap = want;
    return 0;
}

void dfree(fastz_ctx* c, DBuf& b) {
    if (!b.p) return;
    if (c->prm.dev_free) c->prm.dev_free(b.p, c->stream, c->prm.alloc_user);
    else cudaFree(b.p);
    b.p = nullptr;
    b.cap = 0;
}

#define AL(buf, bytes)                               \
    do {                                             \
        int _r = dalloc(c, c->buf, (size_t)(bytes)); \
        if (_r) return _r;                           \
    } while (0)

template <class T>
T* P_(DBuf& b) {
    return reinterpret_cast<T*>(b.p);
}

bool is_device_ptr(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

int check_params(const fastz_params* p) {
    if (!p) return fail(FASTZ_EINVAL, "params is NULL");
    for (int k = 0; k < 16; ++k)
        if (p->sub[k] < -32767 || p->sub[k] > 32767) return fail(FASTZ_EINVAL, "|sub| must be <= 32767");
    if (p->n_score < -32767 || p->n_score > 32767) return fail(FASTZ_EINVAL, "|n_score| must be <= 32767");
    if (p->gap_open < 0 || p->gap_open > (1 << 24)) return fail(FASTZ_EINVAL, "gap_open must be in [0, 2^24]");
    if (p->gap_extend < 1 || p->gap_extend > (1 << 24)) return fail(FASTZ_EINVAL, "gap_extend must be in [1, 2^24]");
    if (p->ydrop < 0 || p->ydrop > (1 << 28)) return fail(FASTZ_EINVAL, "ydrop must be in [0, 2^28]");
    if (p->eager_max < 1 || p->eager_max > 16) return fail(FASTZ_EINVAL, "eager_max must be in [1, 16]");
    return 0;
}

int upload_seq(fastz_ctx* c, const char* src, int64_t len, DBuf& fwd, DBuf& rev, DBuf& fwdn, DBuf& revn,
               bool& has_n, int64_t base_index, int revcomp) {
    const size_t words = (size_t)((len + 15) / 16) + 4;
    int r;
    if ((r = dalloc(c, fwd, words * 4))) return r;
    if ((r = dalloc(c, rev, words * 4))) return r;
    if ((r = dalloc(c, fwdn, words * 2))) return r;
    if ((r = dalloc(c, revn, words * 2))) return r;
    CK(cudaMemsetAsync(fwd.p, 0, words * 4, c->stream));
    CK(cudaMemsetAsync(rev.p, 0, words * 4, c->stream));
    CK(cudaMemsetAsync(fwdn.p, 0, words * 2, c->stream));
    CK(cudaMemsetAsync(revn.p, 0, words * 2, c->stream));
    has_n = false;
    if (len == 0) return 0;
    const char* dsrc = src;
    if (!is_device_ptr(src)) {
        if ((r = dalloc(c, c->stage, (size_t)len))) return r;
        CK(cudaMemcpyAsync(c->stage.p, src, (size_t)len, cudaMemcpyHostToDevice, c->stream));
        dsrc = P_<char>(c->stage);
    }
    if ((r = dalloc(c, c->small, 64))) return r;
    long long init[2] = {LLONG_MAX, 0};  // first invalid character, has-N flag
    CK(cudaMemcpyAsync(c->small.p, init, sizeof(init), cudaMemcpyHostToDevice, c->stream));
    CK(launch_pack(dsrc, len, P_<uint32_t>(fwd), P_<uint32_t>(rev), P_<uint16_t>(fwdn), P_<uint16_t>(revn),
                   P_<long long>(c->small), revcomp, c->stream));
    long long res[2] = {0, 0};
    CK(cudaMemcpyAsync(res, c->small.p, sizeof(res), cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    const long long bad = res[0];
    has_n = res[1] != 0;
    if (bad != LLONG_MAX)
        return fail(FASTZ_EBASE, "invalid base character at index " + std::to_string(base_index + bad) +
                                     (base_index ? " (query offset " + std::to_string(bad) + ")" : " (target)"));
    return 0;
}

int next_pow2(int64_t v) {
    int64_t p = 1;
    while (p < v) p <<= 1;
    return (int)p;
}

Batch make_batch(fastz_ctx* c) {
    Batch b;
    b.Tf = P_<uint32_t>(c->Tf);
    b.Tr = P_<uint32_t>(c->Tr);
    b.Qf = P_<uint32_t>(c->Qf);
    b.Qr = P_<uint32_t>(c->Qr);
    b.TfN = c->t_has_n ? P_<uint16_t>(c->TfN) : nullptr;
    b.TrN = c->t_has_n ? P_<uint16_t>(c->TrN) : nullptr;
    b.QfN = c->q_has_n ? P_<uint16_t>(c->QfN) : nullptr;
    b.QrN = c->q_has_n ? P_<uint16_t>(c->QrN) : nullptr;
    b.tlen = c->tlen;
    b.qlen = c->qlen;
    b.seeds = P_<long long>(c->seeds);
    b.nseeds = (int)c->n;
    return b;
}

SideArrays make_sides(fastz_ctx* c) {
    SideArrays s;
    s.score = P_<int>(c->score);
    s.ti = P_<int>(c->ti);
    s.qj = P_<int>(c->qj);
    s.flags = P_<uint32_t>(c->flags);
    s.eops = P_<unsigned long long>(c->eops);
    s.bound = P_<long long>(c->bound);
    s.maxsw = P_<int>(c->maxsw);
    s.nstrip = P_<int>(c->nstrip);
    return s;
}

ExecPlan make_plan(fastz_ctx* c) {
    ExecPlan p;
    p.woff = P_<long long>(c->woff);
    p.soff = P_<long long>(c->soff);
    p.roff = P_<long long>(c->roff);
    p.bin = P_<int>(c->bin);
    p.list = P_<int>(c->list);
    p.counters = P_<int>(c->counters);
    p.totals = P_<long long>(c->totals);
    p.esc = P_<int>(c->esc);
    p.wl = P_<long long>(c->wl);
    p.wlo = P_<long long>(c->wlo);
    p.wide = P_<int>(c->wide);
    p.redo = P_<int>(c->redo);
    return p;
}

Outputs make_out(fastz_ctx* c) {
    Outputs o;
    o.codes = P_<uint32_t>(c->codes);
    o.stab = P_<int2>(c->stab);
    o.runs = P_<uint32_t>(c->runs);
    o.nruns = P_<int>(c->nruns);
    o.cig_len = P_<long long>(c->ciglen);
    o.cigar = P_<char>(c->cigar);
    o.recs = c->recs.p;
    return o;
}

// Constants of the packed inspector (pair.cuh).  Stored 16-bit value = true + Z.
// Every quantity of a cell must stay in [0, 65535] without any cross-half carry:
//   dead X = NEG_b = max(Y, O+E, E)   (so S - Y, S - OE and D - E never go below 0)
//   NEG_t  = -(Y + 2 + max(sub + OE)) (a cell fed only by dead cells stays below every threshold >= -(Y+1))
//   BIG_b  = NEG_b + 32767            (rows beyond M / columns beyond N; S - W + 0x8000 stays in 16 bits)
//   a side is abandoned (redone in 32 bits) once its peak X reaches limX: values never exceed BIG_b before that
// Returns false when the parameters leave no useful score range (the 32-bit inspector then takes every side).
bool pair_params(const DevParams& d, PairParams& q) {
    int svmax = INT_MIN, svmin = INT_MAX;
    for (int code = 0; code < 5; ++code)
        for (int a = 0; a < 4; ++a) {
            svmax = std::max(svmax, d.sv[5 * code + a]);
            svmin = std::min(svmin, d.sv[5 * code + a]);
        }
    if (d.Y < 0 || d.E < 0 || d.OE < 0 || svmin < 0) return false;
    const int64_t negb = std::max<int64_t>(std::max<int64_t>(d.Y, d.OE), std::max<int64_t>(d.E, 1));
    if (negb > 30000 || svmax > 4000) return false;
    const int64_t bigb = negb + 32767;
    const int64_t negt = -((int64_t)d.Y + 2 + svmax);
    const int64_t Z = negb - negt;
    const int64_t bigt = bigb - Z;
    const int64_t sm = std::max<int64_t>(0, svmax - d.OE);  // largest per-step growth of S
    // peak X (true) that abandons the side: the peak test runs every 2 steps but the half is abandoned at the next
    // 32-step block boundary, so the margin covers 40 steps of growth -- no value of the half ever reaches BIG_t
    // (which keeps S - W + 0x8000 and every add inside the half: no carry into the other side's half)
    const int64_t limt = bigt - d.OE - 40 * sm - 64;
    if (limt < 2000) return false;
    q.Z = (unsigned)Z;
    q.NEGb = (unsigned)negb;
    q.BIGb = (unsigned)bigb;
    q.mE2 = ((65536u - (unsigned)d.E) & 0xffffu) * 0x10001u;
    q.mY2 = 0u - (unsigned)d.Y * 0x10001u;
    q.mOE2 = 0u - (unsigned)d.OE * 0x10001u;
    q.limX = (unsigned)(limt + Z);
    q.WoutT = -d.Y - 1;
    const char* e = getenv("FASTZ_PAIR_ESCAPE");
    q.esc_strips = e ? std::max(1, atoi(e)) : 16;
    q.hist = nullptr;
    return true;
}

// the packed inspector takes this batch: parameters admit it, 4 rows per lane, no N (the N-aware tables are
// 32-bit only), and enough sides to keep every warp busy -- a batch with fewer sides than ~16 per warp is bound by
// its longest sides, which a packed warp steps ~2x slower (FASTZ_PAIR=0 never, =2 always, e.g. for tests)
bool use_pair(const fastz_ctx* c, const Batch& b, int64_t ns) {
    const char* e = getenv("FASTZ_PAIR");
    const int mode = e ? atoi(e) : 1;
    if (mode == 0 || !c->pair_params_ok || c->R != 4 || b.TfN || b.TrN || b.QfN || b.QrN) return false;
    return mode == 2 || ns >= 16 * (int64_t)c->grid_mixed * WARPS;
}

// predicted length (k_predict's ungapped walk, bases) from which a side goes to the 32-bit inspector first
unsigned pair_long_threshold() {
    const char* e = getenv("FASTZ_PAIR_LONG");
    const long v = e ? atol(e) : 32;  // swept on C2/C3/C5/C6 (profiles/r2/pair_sweep.jsonl): 24-32 best
    return (unsigned)(v < 0 ? 0 : v);
}

int ensure_ring(fastz_ctx* c) {
    if (c->ring.p) return 0;
    int r;
    const size_t bytes = (size_t)c->nslots * (size_t)(c->rmask + 1) * sizeof(int4);
    if ((r = dalloc(c, c->ring, bytes))) return r;
    return 0;
}

}  // namespace

extern "C" {

void fastz_default_params(fastz_params* p) {
    static const int32_t hoxd70[16] = {91, -114, -31, -123, -114, 100, -125, -31,
                                       -31, -125, 100, -114, -123, -31, -114, 91};
    memset(p, 0, sizeof(*p));
    memcpy(p->sub, hoxd70, sizeof(hoxd70));
    p->gap_open = 400;
    p->gap_extend = 30;
    p->ydrop = 9400;
    p->gapped_threshold = 3000;
    p->eager_max = 16;
    p->n_score = -100;  // reading R13
}

void fastz_default_seed_params(fastz_seed_params* sp) {
    memset(sp, 0, sizeof(*sp));
    strcpy(sp->pattern, "1110100110010101111");  // 12of19 (LASTZ default [ext]; 19-bp seeds)
    sp->transitions = 1;
    sp->xdrop = 910;
    sp->hspthresh = 3000;
}

const char* fastz_strerror(int status) {
    static thread_local std::string s;
    const char* base = "unknown status";
    switch (status) {
        case FASTZ_OK: base = "ok"; break;
        case FASTZ_EINVAL: base = "invalid argument"; break;
        case FASTZ_EBASE: base = "invalid base character"; break;
        case FASTZ_ERANGE: base = "value out of range"; break;
        case FASTZ_ENOMEM: base = "out of device memory"; break;
        case FASTZ_ECUDA: base = "CUDA error"; break;
        case FASTZ_ETRUNC: base = "output buffer too small"; break;
        case FASTZ_ESTATE: base = "call out of order"; break;
    }
    s = base;
    if (status != FASTZ_OK && !g_err.empty()) s += ": " + g_err;
    return s.c_str();
}

void fastz_destroy(fastz_ctx* c) {
    if (!c) return;
    cudaSetDevice(c->device);
    if (c->stream) cudaStreamSynchronize(c->stream);
    DBuf* bufs[] = {&c->Tf, &c->Tr, &c->Qf, &c->Qr, &c->TfN, &c->TrN, &c->QfN, &c->QrN, &c->stage, &c->seeds, &c->score, &c->ti, &c->qj,
                    &c->flags, &c->eops, &c->bound, &c->maxsw, &c->esc, &c->nstrip, &c->woff, &c->soff, &c->roff, &c->bin, &c->list,
                    &c->counters, &c->totals, &c->tmpa, &c->tmpb, &c->tmpc, &c->scan_tmp, &c->wl, &c->wlo, &c->codes,
                    &c->stab, &c->runs, &c->nruns, &c->ciglen, &c->cigar, &c->recs, &c->cells, &c->ring,
                    &c->wide, &c->ring2, &c->lpt_tmp, &c->order_tmp, &c->order_buf,
                    &c->small, &c->s_kin, &c->s_kout, &c->s_pin, &c->s_pout, &c->s_start, &c->s_cnt, &c->s_off,
                    &c->s_hits, &c->s_hsp, &c->s_keep, &c->s_sel, &c->s_list, &c->s_list2, &c->s_k1, &c->s_k2,
                    &c->s_i1, &c->s_i2, &c->s_flag, &c->s_pos, &c->s_out, &c->s_anch, &c->s_tmp,
                    &c->r_k1, &c->r_k2, &c->r_i1, &c->r_i2, &c->r_box, &c->r_sc, &c->r_red, &c->r_tmp, &c->r_cnt,
                    &c->ring_pair, &c->redo, &c->pdbg, &c->phist};
    for (DBuf* b : bufs) dfree(c, *b);
    if (c->ev_ok)
        for (auto& e : c->ev) cudaEventDestroy(e);
    if (c->own_stream && c->stream) cudaStreamDestroy(c->stream);
    if (c->side_stream) cudaStreamDestroy(c->side_stream);
    if (c->fork_ev) cudaEventDestroy(c->fork_ev);
    if (c->join_ev) cudaEventDestroy(c->join_ev);
    delete c;
}

}  // extern "C"

namespace {

// context with parameters and stream, no sequences yet
int ctx_begin(const fastz_params* p, int64_t tlen, int64_t qlen, int device, void* cuda_stream, fastz_ctx** out) {
    if (!out) return fail(FASTZ_EINVAL, "out is NULL");
    *out = nullptr;
    int r;
    if ((r = check_params(p))) return r;
    if (tlen < 0 || qlen < 0 || tlen >= (1LL << 31) || qlen >= (1LL << 31))
        return fail(FASTZ_ERANGE, "sequence lengths must be in [0, 2^31)");
    CK(cudaSetDevice(device));
    fastz_ctx* c = new fastz_ctx();
    c->device = device;
    c->prm = *p;
    if (cuda_stream) {
        c->stream = (cudaStream_t)cuda_stream;
    } else {
        // a blocking stream: it is ordered after work on the legacy default stream (PyTorch's default), so
        // device inputs written there (seeds, sequences) are complete before the library reads them
        cudaError_t e = cudaStreamCreateWithFlags(&c->stream, cudaStreamDefault);
        if (e != cudaSuccess) {
            delete c;
            return fail(FASTZ_ECUDA, std::string("cudaStreamCreate: ") + cudaGetErrorString(e));
        }
        c->own_stream = true;
    }
    // substitution table with O+E folded in (H = X_diag + v is one FMA-pipe IMAD): sv[5 * code + a], column
    // code 0..3 = query base, 4 = the origin column (sub = 0), 5 = N; target base a = 0..3, 4 = N (R13)
    {
        const int oe = p->gap_open + p->gap_extend;
        for (int code = 0; code < 6; ++code)
            for (int a = 0; a < 5; ++a) {
                int v;
                if (code == 4) v = 0;
                else if (code == 5 || a == 4) v = p->n_score;
                else v = p->sub[4 * a + code];
                c->dp.sv[5 * code + a] = v + oe;
            }
        c->dp.one = 1;
        c->dp.zero = 0;
        c->dp.options = p->options;
    }
    c->dp.O = p->gap_open;
    c->dp.E = p->gap_extend;
    c->dp.Y = p->ydrop;
    c->dp.OE = p->gap_open + p->gap_extend;
    c->dp.K = p->gapped_threshold;
    c->dp.eager_max = p->eager_max;
    c->pair_params_ok = pair_params(c->dp, c->pq);
    c->tlen = (int)tlen;
    c->qlen = (int)qlen;
    *out = c;
    return 0;
}

// launch geometry, boundary rings, events
void ctx_finish(fastz_ctx* c) {
    c->R = pick_R();
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device);
    c->grid = sms * inspector_blocks_per_sm(c->R);
    c->nslots = c->grid * WARPS;
    c->grid_mixed = sms * mixed_blocks_per_sm();
    // per-warp boundary ring: the widest explored band is bounded by the query side length; capped (wider
    // bands take the wide ring, fastz_extend_seeds)
    int64_t want = std::max<int64_t>(std::max<int64_t>(c->tlen, c->qlen) + 64, 1024);
    c->rmask = next_pow2(std::min<int64_t>(want, 1 << 15)) - 1;
    if (const char* e = getenv("FASTZ_RING_ENTRIES"))  // tests: a small ring exercises the wide-band path
        c->rmask = next_pow2(std::max<int64_t>(atoll(e), 64)) - 1;
    for (auto& e : c->ev) cudaEventCreate(&e);
    c->ev_ok = true;
}

// packed (2-bit words + N mask, device memory) -> the context's forward and reversed copies
int upload_packed(fastz_ctx* c, const uint32_t* words, const uint16_t* nmask, int64_t len, DBuf& fwd, DBuf& rev,
                  DBuf& fwdn, DBuf& revn, bool& has_n) {
    const size_t words_n = (size_t)((len + 15) / 16) + 4;
    const size_t used = (size_t)((len + 15) / 16);
    int r;
    if ((r = dalloc(c, fwd, words_n * 4))) return r;
    if ((r = dalloc(c, rev, words_n * 4))) return r;
    if ((r = dalloc(c, fwdn, words_n * 2))) return r;
    if ((r = dalloc(c, revn, words_n * 2))) return r;
    CK(cudaMemsetAsync(fwd.p, 0, words_n * 4, c->stream));
    CK(cudaMemsetAsync(rev.p, 0, words_n * 4, c->stream));
    CK(cudaMemsetAsync(fwdn.p, 0, words_n * 2, c->stream));
    CK(cudaMemsetAsync(revn.p, 0, words_n * 2, c->stream));
    has_n = false;
    if (len == 0) return 0;
    if (!is_device_ptr(words) || (nmask && !is_device_ptr(nmask)))
        return fail(FASTZ_EINVAL, "packed sequences must be device memory");
    CK(cudaMemcpyAsync(fwd.p, words, used * 4, cudaMemcpyDeviceToDevice, c->stream));
    // bases past len in the last word must be 0 (the kernels read whole words)
    if (len % 16) {
        const uint32_t keep = (1u << (2 * (len % 16))) - 1u;
        uint32_t last = 0;
        CK(cudaMemcpyAsync(&last, words + used - 1, 4, cudaMemcpyDeviceToHost, c->stream));
        CK(cudaStreamSynchronize(c->stream));
        last &= keep;
        CK(cudaMemcpyAsync(P_<uint32_t>(fwd) + used - 1, &last, 4, cudaMemcpyHostToDevice, c->stream));
    }
    if (nmask) CK(cudaMemcpyAsync(fwdn.p, nmask, used * 2, cudaMemcpyDeviceToDevice, c->stream));
    if ((r = dalloc(c, c->small, 64))) return r;
    CK(cudaMemsetAsync(c->small.p, 0, 4, c->stream));
    CK(launch_reverse_packed(P_<uint32_t>(fwd), nmask ? P_<uint16_t>(fwdn) : nullptr, len, P_<uint32_t>(rev),
                             P_<uint16_t>(revn), P_<int>(c->small), c->stream));
    int hn = 0;
    CK(cudaMemcpyAsync(&hn, c->small.p, 4, cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    has_n = hn != 0;
    return 0;
}

}  // namespace

extern "C" {

int fastz_create(const fastz_params* p, const char* target, int64_t tlen, const char* query, int64_t qlen,
                 int device, void* cuda_stream, fastz_ctx** out) {
    if ((!target && tlen > 0) || (!query && qlen > 0)) return fail(FASTZ_EINVAL, "sequence pointer is NULL");
    fastz_ctx* c = nullptr;
    int r;
    if ((r = ctx_begin(p, tlen, qlen, device, cuda_stream, &c))) return r;
    if ((r = upload_seq(c, target, tlen, c->Tf, c->Tr, c->TfN, c->TrN, c->t_has_n, 0, 0)) ||
        (r = upload_seq(c, query, qlen, c->Qf, c->Qr, c->QfN, c->QrN, c->q_has_n, tlen,
                        (p->options & FASTZ_OPT_QUERY_REVCOMP) ? 1 : 0))) {
        fastz_destroy(c);
        return r;
    }
    dfree(c, c->stage);
    ctx_finish(c);
    *out = c;
    return 0;
}

int fastz_create_packed(const fastz_params* p, const uint32_t* t_words, const uint16_t* t_nmask, int64_t tlen,
                        const uint32_t* q_words, const uint16_t* q_nmask, int64_t qlen, int device, void* cuda_stream,
                        fastz_ctx** out) {
    if ((!t_words && tlen > 0) || (!q_words && qlen > 0)) return fail(FASTZ_EINVAL, "sequence pointer is NULL");
    fastz_ctx* c = nullptr;
    int r;
    if ((r = ctx_begin(p, tlen, qlen, device, cuda_stream, &c))) return r;
    if ((r = upload_packed(c, t_words, t_nmask, tlen, c->Tf, c->Tr, c->TfN, c->TrN, c->t_has_n)) ||
        (r = upload_packed(c, q_words, q_nmask, qlen, c->Qf, c->Qr, c->QfN, c->QrN, c->q_has_n))) {
        fastz_destroy(c);
        return r;
    }
    ctx_finish(c);
    *out = c;
    return 0;
}

int fastz_pack_sequence(const char* seq, int64_t len, int revcomp, uint32_t* words, uint16_t* nmask, int* has_n,
                        int device, void* cuda_stream) {
    if ((!seq && len > 0) || (len > 0 && (!words || !nmask))) return fail(FASTZ_EINVAL, "NULL argument");
    if (len < 0 || len >= (1LL << 31)) return fail(FASTZ_ERANGE, "length must be in [0, 2^31)");
    CK(cudaSetDevice(device));
    if (has_n) *has_n = 0;
    if (len == 0) return 0;
    if (!is_device_ptr(words) || !is_device_ptr(nmask)) return fail(FASTZ_EINVAL, "words/nmask must be device memory");
    cudaStream_t st = (cudaStream_t)cuda_stream;
    struct Scratch {  // released on every return path
        void* p = nullptr;
        cudaStream_t s = nullptr;
        ~Scratch() {
            if (s) cudaStreamSynchronize(s);
            if (p) cudaFree(p);
        }
    } sc;
    sc.s = st;
    const char* dsrc = seq;
    const size_t nw = (size_t)((len + 15) / 16);
    const bool host = !is_device_ptr(seq);
    CK(cudaMalloc(&sc.p, 64 + (host ? (size_t)len : 0) + nw * 8));
    char* base = static_cast<char*>(sc.p);
    long long* flags = reinterpret_cast<long long*>(base);
    uint32_t* rev = reinterpret_cast<uint32_t*>(base + 64 + (host ? (size_t)len : 0));
    uint16_t* revn = reinterpret_cast<uint16_t*>(rev + nw);
    if (host) {
        CK(cudaMemcpyAsync(base + 64, seq, (size_t)len, cudaMemcpyHostToDevice, st));
        dsrc = base + 64;
    }
    long long init[2] = {LLONG_MAX, 0};
    CK(cudaMemcpyAsync(flags, init, sizeof(init), cudaMemcpyHostToDevice, st));
    CK(launch_pack(dsrc, len, words, rev, nmask, revn, flags, revcomp, st));
    long long res[2] = {0, 0};
    CK(cudaMemcpyAsync(res, flags, sizeof(res), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (res[0] != LLONG_MAX) return fail(FASTZ_EBASE, "invalid base character at index " + std::to_string(res[0]));
    if (has_n) *has_n = res[1] != 0;
    return 0;
}

int fastz_get_packed(fastz_ctx* c, int which, const uint32_t** words, const uint16_t** nmask, int64_t* len) {
    if (!c || (which != 0 && which != 1)) return fail(FASTZ_EINVAL, "bad argument");
    if (words) *words = P_<uint32_t>(which ? c->Qf : c->Tf);
    if (nmask) *nmask = (which ? c->q_has_n : c->t_has_n) ? P_<uint16_t>(which ? c->QfN : c->TfN) : nullptr;
    if (len) *len = which ? c->qlen : c->tlen;
    return 0;
}

int fastz_extend_seeds(fastz_ctx* c, const fastz_seed* seeds, int64_t n, int seeds_on_device) {
    if (!c) return fail(FASTZ_EINVAL, "ctx is NULL");
    if (n < 0 || n > (1 << 29)) return fail(FASTZ_ERANGE, "n must be in [0, 2^29]");
    if (n > 0 && !seeds) return fail(FASTZ_EINVAL, "seeds is NULL");
    CK(cudaSetDevice(c->device));
    Nvtx range_call("fastz_extend_seeds");
    c->have = false;
    c->n = n;
    const int64_t ns = 2 * n;
    cudaStream_t st = c->stream;
    int r;
    if ((r = ensure_ring(c))) return r;
    AL(seeds, std::max<int64_t>(n, 1) * 16);
    AL(score, std::max<int64_t>(ns, 1) * 4);
    AL(ti, std::max<int64_t>(ns, 1) * 4);
    AL(qj, std::max<int64_t>(ns, 1) * 4);
    AL(flags, std::max<int64_t>(ns, 1) * 4);
    AL(eops, std::max<int64_t>(ns, 1) * 8);
    AL(bound, std::max<int64_t>(ns, 1) * 8);
    AL(maxsw, std::max<int64_t>(ns, 1) * 4);
    AL(esc, std::max<int64_t>(ns, 1) * 4);
    AL(redo, std::max<int64_t>(ns, 1) * 4);
    AL(nstrip, std::max<int64_t>(ns, 1) * 4);
    AL(woff, std::max<int64_t>(ns, 1) * 8);
    AL(soff, std::max<int64_t>(ns, 1) * 8);
    AL(roff, std::max<int64_t>(ns, 1) * 8);
    AL(bin, std::max<int64_t>(ns, 1) * 4);
    AL(list, std::max<int64_t>(ns, 1) * 4);
    AL(tmpa, std::max<int64_t>(ns, 1) * 8);
    AL(tmpb, std::max<int64_t>(ns, 1) * 8);
    AL(tmpc, std::max<int64_t>(ns, 1) * 8);
    AL(wl, std::max<int64_t>(ns, 1) * 8);
    AL(wlo, std::max<int64_t>(ns, 1) * 8);
    AL(nruns, std::max<int64_t>(ns, 1) * 4);
    AL(wide, std::max<int64_t>(ns, 1) * 4);
    AL(ciglen, std::max<int64_t>(2 * n, 1) * 8);
    AL(recs, std::max<int64_t>(n, 1) * sizeof(fastz_alignment));
    AL(counters, 96 * 4);
    AL(totals, 8 * 8);
    AL(small, 64);
    const size_t stb = scan_tmp_bytes((int)std::max<int64_t>(ns, 1));
    AL(scan_tmp, stb);

    CK(cudaEventRecord(c->ev[0], st));
    if (n > 0)
        CK(cudaMemcpyAsync(c->seeds.p, seeds, (size_t)n * 16,
                           seeds_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, st));
    CK(cudaMemsetAsync(c->counters.p, 0, 96 * 4, st));
    CK(cudaMemsetAsync(c->totals.p, 0, 8 * 8, st));
    long long init = LLONG_MAX;
    CK(cudaMemcpyAsync(c->small.p, &init, sizeof(init), cudaMemcpyHostToDevice, st));
    Batch b = make_batch(c);
    CK(launch_validate_seeds(b.seeds, b.nseeds, b.tlen, b.qlen, P_<long long>(c->small), st));
    CK(cudaEventRecord(c->ev[1], st));
    Nvtx range_insp("fastz: inspector");

    SideArrays sa = make_sides(c);
    ExecPlan pl = make_plan(c);
    const int esc = (c->dp.options & OPT_NO_BLOCK) ? 0 : escalate_strips();
    c->nwide = 0;
    if (getenv("FASTZ_TEST_SELFCHECK")) c->dp.options |= OPT_SELFCHECK_TEST;  // tests: the self-check must fire
    else c->dp.options &= ~OPT_SELFCHECK_TEST;
    // experiment (FASTZ_L2_PERSIST=1): keep the boundary rings in a persisting L2 window during the inspector
    const bool persist = getenv("FASTZ_L2_PERSIST") != nullptr;
    if (persist) {
        int maxp = 0, maxw = 0;
        cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, c->device);
        cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, c->device);
        const size_t ringb = (size_t)c->nslots * (size_t)(c->rmask + 1) * sizeof(int4);
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min<size_t>((size_t)maxp, ringb));
        cudaStreamAttrValue a{};
        a.accessPolicyWindow.base_ptr = c->ring.p;
        a.accessPolicyWindow.num_bytes = std::min<size_t>(ringb, (size_t)maxw);
        a.accessPolicyWindow.hitRatio = std::min(1.0f, (float)maxp / (float)a.accessPolicyWindow.num_bytes);
        a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a);
        if (getenv("FASTZ_VERBOSE"))
            fprintf(stderr, "L2 persist: max set-aside %d B, max window %d B, ring %zu B, hitRatio %.3f\n", maxp, maxw,
                    ringb, a.accessPolicyWindow.hitRatio);
    }
    // inspector order: predicted-longest sides first (FASTZ_INSPECT_ORDER=0: seed order)
    int* order = nullptr;
    bool ordered = false;
    {
        const char* e = getenv("FASTZ_INSPECT_ORDER");
        ordered = ns > 1 && !(e && atoi(e) == 0);
    }
    if (ordered) {
        const size_t ob = order_tmp_bytes((int)ns);
        AL(order_tmp, ob);
        AL(order_buf, (size_t)ns * 4);
        // keys in/out in tmpa (2 x u32 per side), values in tmpb (the binning scratch is free until launch_bin)
        unsigned* kin = reinterpret_cast<unsigned*>(P_<long long>(c->tmpa));
        CK(launch_order(b, c->dp, (int)ns, kin, kin + ns, P_<int>(c->tmpb), P_<int>(c->order_buf), c->order_tmp.p,
                        c->order_tmp.cap, st));
        order = P_<int>(c->order_buf);
    }
    int64_t pair_launches = 0;
    bool pair_run = false;
    c->n_pair_sides = c->n_redo_sides = c->n_long_sides = 0;
    if (use_pair(c, b, ns)) {
        // Packed inspector (pair.cuh, kernels.cu k_inspect_mixed).  The sides predicted long (k_predict >=
        // FASTZ_PAIR_LONG bases: the head of the order, counted by k_split) run in k_inspect on a second stream,
        // concurrently; the rest run two per warp in 16-bit halves, and the sides the packed inspector abandons
        // (value cap, too many strips) are re-inspected by its own 32-bit path.  The eager walk of the packed sides
        // follows (k_eager).
        int nlong = 0;
        if (ordered) {
            CK(launch_split(reinterpret_cast<unsigned*>(P_<long long>(c->tmpa)) + ns, (int)ns, pair_long_threshold(),
                            P_<int>(c->counters) + 28, st));
            CK(cudaMemcpyAsync(&nlong, P_<int>(c->counters) + 28, 4, cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            pair_launches += 1;
        }
        CK(cudaMemsetAsync(c->redo.p, 0xff, (size_t)ns * 4, st));
        const size_t rb = (size_t)c->grid_mixed * WARPS * (size_t)(c->rmask + 1) * sizeof(int4);
        AL(ring_pair, rb);
        // diagnostics (FASTZ_PAIR_DEBUG=1): per packed side {cycles, strips, steps, redo} -> stderr summary
        long long* dbg = nullptr;
        const bool pdebug = getenv("FASTZ_PAIR_DEBUG") != nullptr;
        if (pdebug) {
            AL(pdbg, (std::max<int64_t>(ns, 1) + (int64_t)c->grid_mixed * WARPS) * 32);
            dbg = P_<long long>(c->pdbg);
            CK(cudaMemsetAsync(dbg, 0, (size_t)(ns + (int64_t)c->grid_mixed * WARPS) * 32, st));
        }
        if (nlong > 0) {
            if (!c->side_stream) {
                CK(cudaStreamCreateWithFlags(&c->side_stream, cudaStreamNonBlocking));
                CK(cudaEventCreateWithFlags(&c->fork_ev, cudaEventDisableTiming));
                CK(cudaEventCreateWithFlags(&c->join_ev, cudaEventDisableTiming));
            }
            CK(cudaEventRecord(c->fork_ev, st));
            CK(cudaStreamWaitEvent(c->side_stream, c->fork_ev, 0));
            CK(launch_inspect(c->R, c->grid, c->dp, b, P_<int4>(c->ring), c->rmask, sa, pl, esc > 0 ? esc : INT_MAX,
                              order, nlong, c->side_stream));
            CK(cudaEventRecord(c->join_ev, c->side_stream));
            pair_launches += 1;
        }
        AL(phist, (size_t)c->grid_mixed * WARPS * 2 * PAIR_HIST * sizeof(int2));
        PairParams pq = c->pq;
        pq.hist = P_<int2>(c->phist);
        CK(launch_inspect_mixed(c->grid_mixed, c->dp, pq, b, P_<int4>(c->ring_pair), c->rmask, sa, pl,
                                ordered ? order : nullptr, (int)ns, nlong, 0, INT_MAX, dbg, st));
        if (nlong > 0) CK(cudaStreamWaitEvent(st, c->join_ev, 0));
        CK(launch_eager(c->dp, b, sa, (int)ns, st));
        pair_launches += 2;
        pair_run = true;
        if (pdebug) {
            const int64_t nw = (int64_t)c->grid_mixed * WARPS;
            std::vector<long long> d((size_t)(ns + nw) * 4);
            CK(cudaMemcpyAsync(d.data(), dbg, (size_t)(ns + nw) * 32, cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            {
                double p1 = 0, p2 = 0, ex = 0, mx1 = 0, mx2 = 0, mxe = 0, n32 = 0;
                for (int64_t w = 0; w < nw; ++w) {
                    const long long* q = &d[(size_t)(4 * ns + 4 * w)];
                    p1 += q[0]; p2 += q[1]; ex += q[2]; n32 += q[3];
                    mx1 = std::max(mx1, (double)q[0]); mx2 = std::max(mx2, (double)q[1]); mxe = std::max(mxe, (double)q[2]);
                }
                fprintf(stderr, "mixed debug: %lld warps; cycles to end of phase 1 mean %.0f max %.0f, phase 2 mean %.0f "
                        "max %.0f, exit mean %.0f max %.0f; 32-bit sides %.0f\n", (long long)nw, p1 / nw, mx1, p2 / nw,
                        mx2, ex / nw, mxe, n32);
            }
            std::vector<int64_t> idx;
            double cyc = 0, steps = 0;
            int64_t nred = 0, npk = 0;
            for (int64_t k = 0; k < ns; ++k)
                if (d[4 * k]) {
                    idx.push_back(k);
                    cyc += (double)d[4 * k];
                    steps += (double)d[4 * k + 2];
                    nred += d[4 * k + 3];
                    ++npk;
                }
            std::sort(idx.begin(), idx.end(), [&](int64_t a, int64_t b2) { return d[4 * a] > d[4 * b2]; });
            fprintf(stderr, "pair debug: %lld packed sides, %lld redo, mean %.0f cycles, mean %.1f steps\n",
                    (long long)npk, (long long)nred, cyc / std::max<int64_t>(npk, 1), steps / std::max<int64_t>(npk, 1));
            for (size_t k = 0; k < idx.size() && k < 8; ++k) {
                const int64_t s2 = idx[k];
                fprintf(stderr, "  side %lld: %lld cycles, %lld strips, %lld steps, redo %lld\n", (long long)s2,
                        d[4 * s2], d[4 * s2 + 1], d[4 * s2 + 2], d[4 * s2 + 3]);
            }
        }
    } else {
        CK(launch_inspect(c->R, c->grid, c->dp, b, P_<int4>(c->ring), c->rmask, sa, pl, esc > 0 ? esc : INT_MAX,
                          order, ordered ? (int)ns : 0, st));
    }
    if (persist) {
        cudaStreamAttrValue a{};
        a.accessPolicyWindow.num_bytes = 0;
        cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a);
        cudaCtxResetPersistingL2Cache();
    }
    if (esc > 0) CK(launch_inspect_block(c->R, c->grid, c->dp, b, P_<int4>(c->ring), c->rmask, sa, pl, st));
    CK(cudaEventRecord(c->ev[2], st));
    range_insp.end();
    Nvtx range_bin("fastz: binning + host sync 1 + pool sizing");
    CK(launch_bin(c->R, c->dp, sa, (int)ns, pl, c->scan_tmp.p, stb, P_<long long>(c->tmpa), P_<long long>(c->tmpb),
                  P_<long long>(c->tmpc), st));
    CK(cudaEventRecord(c->ev[3], st));

    // host sync 1: sizes of the executor's traceback pool
    struct {
        long long totals[5];
        int counters[36];
        long long bad;
    } h;
    auto sync1 = [&]() -> int {
        CK(cudaMemcpyAsync(h.totals, c->totals.p, sizeof(h.totals), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(h.counters, c->counters.p, sizeof(h.counters), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(&h.bad, c->small.p, sizeof(h.bad), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        return 0;
    };
    if ((r = sync1())) return r;
    if (pair_run) {
        c->n_long_sides = ordered ? h.counters[28] : 0;
        c->n_pair_sides = ns - c->n_long_sides;
        c->n_redo_sides = h.counters[30];
    }
    if (h.bad != LLONG_MAX) return fail(FASTZ_ERANGE, "seed " + std::to_string(h.bad) + " lies outside the sequences");
    // Sides whose explored band outgrew the per-warp boundary ring (possible only for very large Y or long
    // indel-rich alignments; the y-drop rule itself has no width limit) are re-inspected with a ring 4x
    // wider, repeatedly, up to the query length (a band never spans more than N + 1 columns); the executor then
    // runs those sides with the same ring.  Memory bounds the number of warp slots of the wide run.
    int64_t extra_launches = 0;
    if (h.counters[20]) {
        int64_t entries = (int64_t)c->rmask + 1;
        const int64_t cap = next_pow2((int64_t)c->qlen + 64);
        for (;;) {
            if (entries >= cap) return fail(FASTZ_ERANGE, "an explored band is wider than the query (internal)");
            entries = std::min<int64_t>(entries * 4, cap);
            const int nw = h.counters[24];
            const size_t slot_bytes = (size_t)entries * sizeof(int4);
            size_t fr = 0, tot = 0;
            cudaMemGetInfo(&fr, &tot);
            const size_t budget = (fr + c->ring2.cap) / 4;
            int64_t slots = (int64_t)(budget / slot_bytes);
            slots = std::min<int64_t>(slots, std::min<int64_t>((int64_t)c->nslots, (int64_t)WARPS * nw));
            const int g2 = (int)(slots / WARPS);
            if (g2 < 1) return fail(FASTZ_ENOMEM, "no memory for a " + std::to_string(slot_bytes) + "-byte wide ring");
            AL(ring2, (size_t)g2 * WARPS * slot_bytes);
            c->grid2 = g2;
            c->rmask2 = (int)(entries - 1);
            // re-inspect the listed sides (wide list -> tmp copy, since binning rebuilds it)
            int* wl = P_<int>(c->tmpc);
            CK(cudaMemcpyAsync(wl, c->wide.p, (size_t)nw * 4, cudaMemcpyDeviceToDevice, st));
            CK(cudaMemsetAsync(c->counters.p, 0, 96 * 4, st));
            CK(launch_inspect(c->R, c->grid2, c->dp, b, P_<int4>(c->ring2), c->rmask2, sa, pl, INT_MAX, wl, nw, st));
            CK(launch_mark_wide(sa, wl, nw, st));
            CK(cudaMemsetAsync(c->counters.p, 0, 96 * 4, st));
            CK(launch_bin(c->R, c->dp, sa, (int)ns, pl, c->scan_tmp.p, stb, P_<long long>(c->tmpa),
                          P_<long long>(c->tmpb), P_<long long>(c->tmpc), st));
            if ((r = sync1())) return r;
            c->nwide = nw;
            extra_launches += 7;  // inspect, mark_wide + bin_count, bin_offsets, bin_scatter, list_words, list_offsets
            if (!h.counters[20]) break;
        }
        // the final wide list: every side inspected with the wide ring (SF_WIDE), for the census
        CK(launch_wide_list(sa, (int)ns, P_<int>(c->wide), P_<int>(c->counters) + 25, st));
        extra_launches += 1;
        int nwl = 0;
        CK(cudaMemcpyAsync(&nwl, P_<int>(c->counters) + 25, 4, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        c->nwide = nwl;
    }
    const long long words = h.totals[0], strips = h.totals[1], nrun = h.totals[2];
    c->nexec = h.totals[3];
    const long long nblock = h.totals[4];
    if (nblock > 1) {  // LPT inside the block-per-side bins; the total words are unchanged
        const size_t lb = lpt_tmp_bytes((int)nblock);
        AL(lpt_tmp, lb);
        CK(launch_lpt(pl, (int)nblock, (int)c->nexec, P_<long long>(c->tmpa), P_<long long>(c->wl),
                      P_<long long>(c->wlo), P_<int>(c->tmpb), c->lpt_tmp.p, c->lpt_tmp.cap, c->scan_tmp.p, stb, st));
        extra_launches += 3;
    }
    AL(stab, std::max<long long>(strips, 1) * 8);
    AL(runs, std::max<long long>(nrun, 1) * 4);
    // traceback-code pool: one wave if it fits the budget, else consecutive ranges of the executor list
    // (largest bins first), each executed and traced back before the pool is reused
    long long budget_words;
    {
        const char* e = getenv("FASTZ_POOL_MB");
        if (e) {
            budget_words = std::max<long long>(atoll(e), 1) * (1LL << 20) / 4;
        } else if (words <= (long long)(c->codes.cap / 4)) {
            budget_words = words;  // the pool already holds one wave: no memory query on the common path
        } else {
            size_t fr = 0, tot = 0;  // cudaMemGetInfo costs milliseconds: only when the pool must grow
            cudaMemGetInfo(&fr, &tot);
            // 80% of what is free (plus the pool itself): waves cost a tail each, so use the memory
            budget_words = (long long)((double)(fr + c->codes.cap) * 0.8 / 4);
        }
    }
    std::vector<std::pair<long long, long long>> waves;  // list ranges [a, b)
    std::vector<long long> wbase;
    long long pool_words = words;
    if (words <= budget_words || c->nexec <= 1) {
        waves.push_back({0, c->nexec});
        wbase.push_back(0);
    } else {
        std::vector<long long> wlo((size_t)c->nexec + 1);
        CK(cudaMemcpyAsync(wlo.data(), c->wlo.p, (size_t)c->nexec * 8, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        wlo[(size_t)c->nexec] = words;
        pool_words = 0;
        long long a = 0;
        while (a < c->nexec) {
            long long b = a + 1;
            while (b < c->nexec && wlo[(size_t)b + 1] - wlo[(size_t)a] <= budget_words) ++b;
            waves.push_back({a, b});
            wbase.push_back(wlo[(size_t)a]);
            pool_words = std::max(pool_words, wlo[(size_t)b] - wlo[(size_t)a]);
            a = b;
        }
    }
    AL(codes, std::max<long long>(pool_words, 1) * 4);
    Outputs o = make_out(c);
    // executor timing starts here: the host sync + pool sizing above count to the binning stage
    CK(cudaEventRecord(c->ev[7], st));
    range_bin.end();
    Nvtx range_exec("fastz: executor + traceback + CIGAR");
    int64_t tb_launches = 0;  // per wave: warp-per-side (list positions < nblock) and thread-per-side launches
    for (size_t w = 0; w < waves.size(); ++w) {
        {
            const long long lo = waves[w].first, hi = waves[w].second;
            const long long mid = std::min(std::max(nblock, lo), hi);
            tb_launches += (mid > lo ? 1 : 0) + (hi > mid ? 1 : 0);
        }
        if (w) CK(cudaMemsetAsync(P_<int>(c->counters) + 1, 0, 4, st));
        if (w) CK(cudaMemsetAsync(P_<int>(c->counters) + 23, 0, 4, st));
        CK(launch_execute(c->R, c->grid, c->dp, b, P_<int4>(c->ring), c->rmask, sa, pl, (int)waves[w].first,
                          (int)waves[w].second, (int)nblock, wbase[w], o, 0, st));
        if (c->nwide) {  // the SF_WIDE sides of this wave, with the wide ring
            CK(cudaMemsetAsync(P_<int>(c->counters) + 1, 0, 4, st));
            CK(cudaMemsetAsync(P_<int>(c->counters) + 23, 0, 4, st));
            CK(launch_execute(c->R, c->grid2, c->dp, b, P_<int4>(c->ring2), c->rmask2, sa, pl, (int)waves[w].first,
                              (int)waves[w].second, (int)nblock, wbase[w], o, 1, st));
            extra_launches += 1;
        }
        if (w == 0) CK(cudaEventRecord(c->ev[4], st));
        CK(launch_traceback(c->R, sa, pl, (int)waves[w].first, (int)waves[w].second, (int)nblock, wbase[w], o, st));
    }
    if (waves.empty()) CK(cudaEventRecord(c->ev[4], st));
    CK(cudaEventRecord(c->ev[5], st));
    c->nwaves = (int)waves.size();
    long long* dtotal = P_<long long>(c->small) + 1;
    CK(launch_combine_len(c->dp, b, sa, pl, o, c->scan_tmp.p, stb, dtotal, st));
    long long ctot = 0;
    int nfail = 0;
    long long h_written = 0;
    CK(cudaMemcpyAsync(&ctot, dtotal, sizeof(ctot), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&h_written, P_<long long>(c->totals) + 6, sizeof(h_written), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&nfail, P_<int>(c->counters) + 26, sizeof(nfail), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));  // host sync 2: CIGAR bytes, executor self-check
    if (nfail)
        return fail(FASTZ_ECUDA, "executor self-check failed on " + std::to_string(nfail) +
                                     " sides (S(i*,j*) differs from the inspector's peak, or a traceback-code store "
                                     "left the side's reservation)");
    AL(cigar, std::max<long long>(ctot, 1));
    o = make_out(c);
    CK(launch_combine_write(c->dp, b, sa, pl, o, st));
    CK(cudaEventRecord(c->ev[6], st));
    c->cigar_bytes = ctot;

    fastz_stats& S = c->stats;
    memset(&S, 0, sizeof(S));
    S.n_warp_slots = c->nslots;
    S.n_seeds = n;
    S.n_sides = ns;
    S.n_exec_sides = c->nexec;
    S.n_eager_sides = h.counters[2];
    for (int k = 0; k < 7; ++k) S.bin_counts[k] = h.counters[2 + k];
    S.exec_words = h_written;
    S.exec_reserved_words = words;
    S.cigar_bytes = ctot;
    S.n_waves = c->nwaves;
    S.n_escalated = h.counters[21];
    // own kernels: validate, inspect, inspect_block (if escalation on), bin_count, bin_offsets, bin_scatter,
    // list_words, list_offsets, execute per wave, traceback (warp and/or thread variant) per wave, combine_len,
    // combine_total, combine_write
    S.n_launches = (n > 0 ? 1 + 1 + (esc > 0 ? 1 : 0) + 5 + (int64_t)c->nwaves + tb_launches + 3 + extra_launches +
                               (ordered ? 1 : 0) + pair_launches : 1);
    S.n_wide_sides = c->nwide;
    S.n_packed_sides = c->n_pair_sides;
    S.n_long_sides = c->n_long_sides;
    S.n_redo_sides = c->n_redo_sides;
    c->have = true;
    return 0;
}

int fastz_get_alignments(fastz_ctx* c, fastz_alignment* out, int64_t out_cap, char* cigar, int64_t cigar_cap,
                         int64_t* n_out, int64_t* cigar_bytes) {
    if (!c) return fail(FASTZ_EINVAL, "ctx is NULL");
    if (!c->have) return fail(FASTZ_ESTATE, "no results: call fastz_extend_seeds first");
    CK(cudaSetDevice(c->device));
    if (n_out) *n_out = c->n;
    if (cigar_bytes) *cigar_bytes = c->cigar_bytes;
    if (out_cap < c->n || cigar_cap < c->cigar_bytes) return fail(FASTZ_ETRUNC, "output buffers too small");
    if ((c->n && !out) || (c->cigar_bytes && !cigar)) return fail(FASTZ_EINVAL, "output pointer is NULL");
    if (c->n) CK(cudaMemcpyAsync(out, c->recs.p, (size_t)c->n * sizeof(fastz_alignment), cudaMemcpyDeviceToHost, c->stream));
    if (c->cigar_bytes) CK(cudaMemcpyAsync(cigar, c->cigar.p, (size_t)c->cigar_bytes, cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    return 0;
}

int fastz_get_alignments_device(fastz_ctx* c, const fastz_alignment** recs, const char** cigar, int64_t* n,
                                int64_t* cigar_bytes) {
    if (!c) return fail(FASTZ_EINVAL, "ctx is NULL");
    if (!c->have) return fail(FASTZ_ESTATE, "no results: call fastz_extend_seeds first");
    if (recs) *recs = reinterpret_cast<const fastz_alignment*>(c->recs.p);
    if (cigar) *cigar = P_<char>(c->cigar);
    if (n) *n = c->n;
    if (cigar_bytes) *cigar_bytes = c->cigar_bytes;
    return 0;
}

int fastz_get_sides(fastz_ctx* c, int32_t* score, int32_t* ti, int32_t* qj, uint32_t* flags, int64_t cap) {
    if (!c) return fail(FASTZ_EINVAL, "ctx is NULL");
    if (!c->have) return fail(FASTZ_ESTATE, "no results: call fastz_extend_seeds first");
    if (cap < 2 * c->n) return fail(FASTZ_ETRUNC, "cap < 2n");
    CK(cudaSetDevice(c->device));
    const size_t bytes = (size_t)(2 * c->n) * 4;
    if (bytes) {
        if (score) CK(cudaMemcpyAsync(score, c->score.p, bytes, cudaMemcpyDeviceToHost, c->stream));
        if (ti) CK(cudaMemcpyAsync(ti, c->ti.p, bytes, cudaMemcpyDeviceToHost, c->stream));
        if (qj) CK(cudaMemcpyAsync(qj, c->qj.p, bytes, cudaMemcpyDeviceToHost, c->stream));
        if (flags) CK(cudaMemcpyAsync(flags, c->flags.p, bytes, cudaMemcpyDeviceToHost, c->stream));
    }
    CK(cudaStreamSynchronize(c->stream));
    if (flags)
        for (int64_t k = 0; k < 2 * c->n; ++k) flags[k] &= 0xffu;
    return 0;
}

int fastz_census(fastz_ctx* c, int64_t* cells, int64_t cap) {
    if (!c) return fail(FASTZ_EINVAL, "ctx is NULL");
    if (!c->have) return fail(FASTZ_ESTATE, "no results: call fastz_extend_seeds first");
    if (cap < 2 * c->n) return fail(FASTZ_ETRUNC, "cap < 2n");
    CK(cudaSetDevice(c->device));
    AL(cells, std::max<int64_t>(2 * c->n, 1) * 8);
    CK(cudaMemsetAsync(c->counters.p, 0, 4, c->stream));
    Batch b = make_batch(c);
    CK(launch_census(c->R, c->grid, c->dp, b, P_<int4>(c->ring), c->rmask, P_<long long>(c->cells),
                     P_<int>(c->counters), nullptr, 0, c->stream));
    if (c->nwide) {  // sides with a band wider than the regular ring: recount with the wide ring
        CK(cudaMemsetAsync(c->counters.p, 0, 4, c->stream));
        CK(launch_census(c->R, c->grid2, c->dp, b, P_<int4>(c->ring2), c->rmask2, P_<long long>(c->cells),
                         P_<int>(c->counters), P_<int>(c->wide), c->nwide, c->stream));
    }
    if (c->n) CK(cudaMemcpyAsync(cells, c->cells.p, (size_t)(2 * c->n) * 8, cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    for (int64_t k = 0; k < 2 * c->n; ++k)
        if (cells[k] < 0) return fail(FASTZ_ERANGE, "an explored band is wider than the per-warp boundary ring");
    return 0;
}

int fastz_get_stats(fastz_ctx* c, fastz_stats* s) {
    if (!c || !s) return fail(FASTZ_EINVAL, "NULL argument");
    if (!c->have) return fail(FASTZ_ESTATE, "no results: call fastz_extend_seeds first");
    CK(cudaEventSynchronize(c->ev[6]));
    fastz_stats& S = c->stats;
    auto el = [&](int a, int b) {
        float ms = 0;
        cudaEventElapsedTime(&ms, c->ev[a], c->ev[b]);
        return ms;
    };
    S.ms_upload = el(0, 1);
    S.ms_inspect = el(1, 2);
    S.ms_bin = el(2, 7);      // binning kernels + host sync 1 + traceback-pool sizing
    S.ms_execute = el(7, 4);
    S.ms_traceback = el(4, 5);
    S.ms_combine = el(5, 6);
    S.ms_total = el(0, 6);
    *s = S;
    return 0;
}

int fastz_mark_redundant(fastz_ctx* c, uint8_t* redundant, int64_t cap, int64_t* n_redundant) {
    if (!c) return fail(FASTZ_EINVAL, "ctx is NULL");
    if (!c->have) return fail(FASTZ_ESTATE, "no results: call fastz_extend_seeds first");
    if (redundant && cap < c->n) return fail(FASTZ_ETRUNC, "cap < n");
    CK(cudaSetDevice(c->device));
    const int n = (int)c->n;
    const size_t m = (size_t)std::max(n, 1);
    const size_t tb = redundant_tmp_bytes(n);
    AL(r_k1, m * 4);
    AL(r_k2, m * 4);
    AL(r_i1, m * 4);
    AL(r_i2, m * 4);
    AL(r_box, m * 16);
    AL(r_sc, m * 8);
    AL(r_red, m);
    AL(r_tmp, tb);
    AL(r_cnt, 16);
    CK(launch_redundant(c->recs.p, n, c->r_tmp.p, c->r_tmp.cap, P_<uint32_t>(c->r_k1), P_<uint32_t>(c->r_k2),
                        P_<int>(c->r_i1), P_<int>(c->r_i2), P_<int4>(c->r_box), P_<int2>(c->r_sc),
                        P_<unsigned char>(c->r_red), P_<int>(c->r_cnt), c->stream));
    int cnt[3] = {0, 0, 0};
    CK(cudaMemcpyAsync(cnt, c->r_cnt.p, sizeof(cnt), cudaMemcpyDeviceToHost, c->stream));
    if (redundant && n) CK(cudaMemcpyAsync(redundant, c->r_red.p, (size_t)n, cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    if (n_redundant) *n_redundant = cnt[2];
    return 0;
}

int fastz_mark_redundant_records(fastz_alignment* recs, int64_t n, int recs_on_device, uint8_t* redundant,
                                 int64_t* n_redundant, int device) {
    if (n < 0 || n > INT_MAX) return fail(FASTZ_EINVAL, "n must be in [0, 2^31)");
    if (n && !recs) return fail(FASTZ_EINVAL, "recs is NULL");
    if (n_redundant) *n_redundant = 0;
    if (n == 0) return 0;
    CK(cudaSetDevice(device));
    struct Scratch {  // released on every return path
        void* p = nullptr;
        cudaStream_t s = nullptr;
        ~Scratch() {
            if (s) cudaStreamSynchronize(s);
            if (p) cudaFree(p);
            if (s) cudaStreamDestroy(s);
        }
    } sc;
    CK(cudaStreamCreateWithFlags(&sc.s, cudaStreamDefault));  // ordered after the legacy default stream
    const size_t m = (size_t)n;
    auto up = [](size_t b) { return (b + 255) & ~(size_t)255; };
    const size_t tb = redundant_tmp_bytes((int)n);
    const size_t o_rec = 0, o_k1 = o_rec + (recs_on_device ? 0 : up(m * sizeof(fastz_alignment)));
    const size_t o_k2 = o_k1 + up(m * 4), o_i1 = o_k2 + up(m * 4), o_i2 = o_i1 + up(m * 4);
    const size_t o_box = o_i2 + up(m * 4), o_sc = o_box + up(m * 16), o_red = o_sc + up(m * 8);
    const size_t o_cnt = o_red + up(m), o_tmp = o_cnt + 256, total = o_tmp + up(tb);
    CK(cudaMalloc(&sc.p, total));
    char* base = static_cast<char*>(sc.p);
    void* drecs = recs_on_device ? (void*)recs : (void*)(base + o_rec);
    if (!recs_on_device)
        CK(cudaMemcpyAsync(drecs, recs, m * sizeof(fastz_alignment), cudaMemcpyHostToDevice, sc.s));
    CK(launch_redundant(drecs, (int)n, base + o_tmp, up(tb), (uint32_t*)(base + o_k1), (uint32_t*)(base + o_k2),
                        (int*)(base + o_i1), (int*)(base + o_i2), (int4*)(base + o_box), (int2*)(base + o_sc),
                        (unsigned char*)(base + o_red), (int*)(base + o_cnt), sc.s));
    int cnt[3] = {0, 0, 0};
    CK(cudaMemcpyAsync(cnt, base + o_cnt, sizeof(cnt), cudaMemcpyDeviceToHost, sc.s));
    if (redundant) CK(cudaMemcpyAsync(redundant, base + o_red, m, cudaMemcpyDeviceToHost, sc.s));
    if (!recs_on_device)
        CK(cudaMemcpyAsync(recs, drecs, m * sizeof(fastz_alignment), cudaMemcpyDeviceToHost, sc.s));
    CK(cudaStreamSynchronize(sc.s));
    if (n_redundant) *n_redundant = cnt[2];
    return 0;
}

int fastz_int_peak(int device, float ms, double* ops_per_s, double* sm_clock_mhz) {
    if (!ops_per_s || !sm_clock_mhz) return fail(FASTZ_EINVAL, "NULL argument");
    CK(int_peak_run(device, ms, ops_per_s, sm_clock_mhz));
    return 0;
}

static_assert(sizeof(HspOut) == sizeof(fastz_hsp), "fastz_hsp layout");

int fastz_find_hsps(fastz_ctx* c, const fastz_seed_params* spp, fastz_hsp* hsps, fastz_seed* anchors, int64_t cap,
                    int64_t* n_out, int64_t* n_hits) {
    if (!c || !spp || !n_out) return fail(FASTZ_EINVAL, "NULL argument");
    if (cap < 0) return fail(FASTZ_EINVAL, "cap < 0");
    // S1: parse the spaced seed
    SeedPattern sp{};
    const size_t L = strnlen(spp->pattern, sizeof(spp->pattern));
    if (L == 0 || L > 32) return fail(FASTZ_EINVAL, "seed pattern span must be 1..32");
    for (size_t i = 0; i < L; ++i) {
        if (spp->pattern[i] == '1') {
            if (sp.w == 16) return fail(FASTZ_EINVAL, "seed pattern has more than 16 care positions");
            sp.caremask |= 1u << i;
            sp.off[sp.w++] = (int)i;
        } else if (spp->pattern[i] != '0') {
            return fail(FASTZ_EINVAL, "seed pattern characters must be '0' or '1'");
        }
    }
    if (spp->pattern[0] != '1' || spp->pattern[L - 1] != '1')
        return fail(FASTZ_EINVAL, "seed pattern must start and end with '1'");
    if (spp->xdrop < 0) return fail(FASTZ_EINVAL, "xdrop must be >= 0");
    sp.L = (int)L;
    UngappedParams up{};
    for (int a = 0; a < 5; ++a)
        for (int b = 0; b < 5; ++b) up.sub[5 * a + b] = (a == 4 || b == 4) ? c->prm.n_score : c->prm.sub[4 * a + b];
    up.xdrop = spp->xdrop;
    up.hspthresh = spp->hspthresh;
    const int nvar = spp->transitions ? 1 + sp.w : 1;
    CK(cudaSetDevice(c->device));
    cudaStream_t st = c->stream;
    const long long nt = c->tlen >= sp.L ? (long long)c->tlen - sp.L + 1 : 0;
    const long long nq = c->qlen >= sp.L ? (long long)c->qlen - sp.L + 1 : 0;
    const long long nkeys = 1LL << (2 * sp.w);
    const bool dense = sp.w <= 12;
    long long HIT_CAP = 1LL << 25;  // hits per query chunk (24 B of scratch each); env override for tests
    if (const char* e = getenv("FASTZ_SEED_HIT_CAP")) HIT_CAP = std::max(1LL, atoll(e));
    long long QC = std::min<long long>(std::max<long long>(nq, 1), std::min(1LL << 22, HIT_CAP));

    // index of the target: (word, position) sorted, dense bucket starts
    const size_t tmpb = seed_sort_tmp_bytes(std::max(std::max(nt, HIT_CAP), QC + 1));
    AL(s_tmp, tmpb);
    AL(s_kin, 4 * (nt + 1));
    AL(s_kout, 4 * (nt + 1));
    AL(s_pin, 4 * (nt + 1));
    AL(s_pout, 4 * (nt + 1));
    if (dense) AL(s_start, 4 * (nkeys + 1));
    AL(s_cnt, 8 * (QC + 1));
    AL(s_off, 8 * (QC + 1));
    const uint16_t* TfN = c->t_has_n ? P_<uint16_t>(c->TfN) : nullptr;
    const uint16_t* QfN = c->q_has_n ? P_<uint16_t>(c->QfN) : nullptr;
    long long ntv = nt;  // target words in the index (S7: words with an N at a care position are dropped)
    if (TfN) {
        AL(s_keep, nt + 1);
        AL(s_flag, 4);
        CK(seed_keys(P_<uint32_t>(c->Tf), TfN, nt, sp, P_<uint32_t>(c->s_kout), P_<int>(c->s_pout),
                     P_<unsigned char>(c->s_keep), st));
        if (nt > 0) {
            CK(seed_compact(c->s_tmp.p, tmpb, P_<uint32_t>(c->s_kout), P_<int>(c->s_pout), P_<unsigned char>(c->s_keep),
                            nt, P_<uint32_t>(c->s_kin), P_<int>(c->s_pin), P_<int>(c->s_flag), st));
            int nv = 0;
            CK(cudaMemcpyAsync(&nv, c->s_flag.p, sizeof(int), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            ntv = nv;
        }
    } else {
        CK(seed_keys(P_<uint32_t>(c->Tf), nullptr, nt, sp, P_<uint32_t>(c->s_kin), P_<int>(c->s_pin), nullptr, st));
    }
    CK(seed_sort_words(c->s_tmp.p, tmpb, P_<uint32_t>(c->s_kin), P_<uint32_t>(c->s_kout), P_<int>(c->s_pin),
                       P_<int>(c->s_pout), ntv, 2 * sp.w, st));
    const int* start = nullptr;
    if (dense) {
        CK(seed_bucket_start(P_<uint32_t>(c->s_kout), ntv, P_<int>(c->s_start), nkeys, st));
        start = P_<int>(c->s_start);
    }
    // query chunks: count -> scan -> (D2H total) -> write hits -> ungapped walks -> select survivors
    long long q0 = 0, hits_total = 0, nlist = 0, list_cap = 0;
    while (q0 < nq) {
        const long long nqc = std::min(QC, nq - q0);
        CK(seed_count(P_<uint32_t>(c->Qf), QfN, q0, nqc, sp, nvar, P_<uint32_t>(c->s_kout), P_<int>(c->s_pout), start, ntv,
                      P_<long long>(c->s_cnt), P_<long long>(c->s_off), c->s_tmp.p, tmpb, st));
        long long nh = 0;
        CK(cudaMemcpyAsync(&nh, P_<long long>(c->s_off) + nqc, sizeof(nh), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        if (nh > HIT_CAP && nqc > 1) {  // too many hits for the scratch: halve the chunk
            QC = std::max<long long>(1, nqc / 2);
            continue;
        }
        if (nh > (1LL << 31) - 1) return fail(FASTZ_ERANGE, "a query word has more than 2^31 seed hits");
        if (nh > 0) {
            AL(s_hits, 8 * nh);
            AL(s_hsp, 16 * nh);
            AL(s_keep, nh);
            AL(s_sel, 16 * nh + 16);
            const size_t tb2 = seed_sort_tmp_bytes(nh);
            if (tb2 > c->s_tmp.cap) AL(s_tmp, tb2);
            CK(seed_write_extend(P_<uint32_t>(c->Tf), P_<uint32_t>(c->Qf), TfN, QfN, c->tlen, c->qlen, q0, nqc, sp, nvar,
                                 P_<uint32_t>(c->s_kout), P_<int>(c->s_pout), start, ntv, P_<long long>(c->s_off), nh,
                                 P_<int2>(c->s_hits), up, P_<int4>(c->s_hsp), P_<unsigned char>(c->s_keep), st));
            int* nsel_d = reinterpret_cast<int*>(P_<int4>(c->s_sel) + nh);
            CK(seed_select(c->s_tmp.p, c->s_tmp.cap, P_<int4>(c->s_hsp), P_<unsigned char>(c->s_keep), nh,
                           P_<int4>(c->s_sel), nsel_d, st));
            int nsel = 0;
            CK(cudaMemcpyAsync(&nsel, nsel_d, sizeof(int), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            if (nsel > 0) {
                if (nlist + nsel > list_cap) {  // grow the HSP list, keeping its contents
                    list_cap = std::max<long long>(2 * list_cap, nlist + nsel);
                    AL(s_list2, 16 * list_cap);
                    if (nlist) CK(cudaMemcpyAsync(c->s_list2.p, c->s_list.p, 16 * nlist, cudaMemcpyDeviceToDevice, st));
                    std::swap(c->s_list, c->s_list2);
                }
                CK(cudaMemcpyAsync(P_<int4>(c->s_list) + nlist, c->s_sel.p, 16 * (size_t)nsel,
                                   cudaMemcpyDeviceToDevice, st));
                nlist += nsel;
            }
        }
        hits_total += nh;
        q0 += nqc;
    }
    if (n_hits) *n_hits = hits_total;
    long long nu = 0;
    if (nlist > 0) {
        AL(s_k1, 8 * nlist);
        AL(s_k2, 16 * nlist);
        AL(s_i1, 4 * nlist);
        AL(s_i2, 4 * nlist);
        AL(s_flag, 4 * (nlist + 1));
        AL(s_pos, 4 * (nlist + 1));
        const size_t tb3 = seed_sort_tmp_bytes(nlist);
        if (tb3 > c->s_tmp.cap) AL(s_tmp, tb3);
        CK(seed_finish_sort(c->s_tmp.p, c->s_tmp.cap, P_<int4>(c->s_list), nlist, P_<unsigned long long>(c->s_k1),
                            P_<unsigned long long>(c->s_k2), P_<int>(c->s_i1), P_<int>(c->s_i2), st));
        AL(s_out, sizeof(HspOut) * nlist);
        AL(s_anch, 16 * nlist);
        CK(seed_unique_emit(c->s_tmp.p, c->s_tmp.cap, P_<int4>(c->s_list), P_<int>(c->s_i1), nlist, P_<int>(c->s_flag),
                            P_<int>(c->s_pos), P_<HspOut>(c->s_out), P_<long long>(c->s_anch), st));
        int nuu = 0;
        CK(cudaMemcpyAsync(&nuu, P_<int>(c->s_pos) + nlist, sizeof(int), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        nu = nuu;
    }
    *n_out = nu;
    if (nu > cap) return fail(FASTZ_ETRUNC, "HSP buffer too small: " + std::to_string(nu) + " needed");
    if (nu > 0 && hsps) CK(cudaMemcpyAsync(hsps, c->s_out.p, sizeof(fastz_hsp) * nu, cudaMemcpyDeviceToHost, st));
    if (nu > 0 && anchors)
        CK(cudaMemcpyAsync(anchors, c->s_anch.p, sizeof(fastz_seed) * nu, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    return 0;
}

}  // extern "C"
