// kernels.cu -- sm_100a kernels of the FastZ hot path: pack, inspector, census, binning, executor,
// traceback, CIGAR assembly.  Citations P:<n> are PAPER.md lines; readings R1..R8 are in DESIGN.md.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include "../../include/fastz.h"
#include "internal.h"
#include "side.cuh"

namespace fz {

// ------------------------------------------------------------------------------------------------- pack
// ASCII -> 2-bit codes (A0 C1 G2 T3, lowercase folded), forward and reversed copies (the left extension
// reads the reversed copies).  One thread per output word of 16 bases.
__device__ __forceinline__ int code_of(unsigned char c) {
    switch (c) {
        case 'A': case 'a': return 0;
        case 'C': case 'c': return 1;
        case 'G': case 'g': return 2;
        case 'T': case 't': return 3;
        case 'N': case 'n': return 4;  // reading R13: packed as 0 plus a bit in the N mask
        default: return -1;
    }
}

__global__ void k_pack(const char* __restrict__ src, long long n, uint32_t* __restrict__ fwd,
                       uint32_t* __restrict__ rev, uint16_t* __restrict__ fwdn, uint16_t* __restrict__ revn,
                       long long* bad, int revcomp) {
    const long long w = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long nw = (n + 15) / 16;
    if (w >= nw) return;
    // revcomp: the sequence is the reverse complement of src (A<->T, C<->G: code xor 3; N stays N), so its
    // forward copy reads src backwards and its reversed copy reads src forwards, both complemented
    const uint32_t cx = revcomp ? 3u : 0u;
    uint32_t f = 0, r = 0, fn = 0, rn = 0;
#pragma unroll 4
    for (int i = 0; i < 16; ++i) {
        const long long p = 16 * w + i;
        if (p < n) {
            const long long pf = revcomp ? n - 1 - p : p;
            int c = code_of((unsigned char)src[pf]);
            if (c < 0) { atomicMin(bad, pf); c = 0; }
            if (c == 4) { fn |= 1u << i; c = 0; }
            f |= ((uint32_t)c ^ cx) << (2 * i);
            int cr = code_of((unsigned char)src[revcomp ? p : n - 1 - p]);
            if (cr < 0) cr = 0;
            if (cr == 4) { rn |= 1u << i; cr = 0; }
            r |= ((uint32_t)cr ^ cx) << (2 * i);
        }
    }
    fwd[w] = f;
    rev[w] = r;
    fwdn[w] = (uint16_t)fn;
    revn[w] = (uint16_t)rn;
    if (fn) atomicOr((unsigned long long*)(bad + 1), 1ull);  // the sequence has an N
}

cudaError_t launch_pack(const char* src, int64_t n, uint32_t* fwd, uint32_t* rev, uint16_t* fwdn, uint16_t* revn,
                        long long* bad, int revcomp, cudaStream_t st) {
    const long long nw = (n + 15) / 16;
    if (nw == 0) return cudaSuccess;
    k_pack<<<(unsigned)((nw + 255) / 256), 256, 0, st>>>(src, n, fwd, rev, fwdn, revn, bad, revcomp);
    return cudaGetLastError();
}

// Reversed copy (and N mask) of a packed sequence: base p of the output is base n-1-p of the input.  Also ORs
// every input mask word into *has_n.  One thread per output word of 16 bases.
__global__ void k_reverse_packed(const uint32_t* __restrict__ fwd, const uint16_t* __restrict__ fwdn, long long n,
                                 uint32_t* __restrict__ rev, uint16_t* __restrict__ revn, int* has_n) {
    const long long w = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long nw = (n + 15) / 16;
    if (w >= nw) return;
    uint32_t r = 0, rn = 0;
    for (int i = 0; i < 16; ++i) {
        const long long p = 16 * w + i;
        if (p < n) {
            const long long q = n - 1 - p;
            r |= ((fwd[q >> 4] >> (2 * (q & 15))) & 3u) << (2 * i);
            if (fwdn) rn |= ((uint32_t)(fwdn[q >> 4] >> (q & 15)) & 1u) << i;
        }
    }
    rev[w] = r;
    revn[w] = (uint16_t)rn;
    if (fwdn && fwdn[w]) atomicOr(has_n, 1);
}

cudaError_t launch_reverse_packed(const uint32_t* fwd, const uint16_t* fwdn, int64_t n, uint32_t* rev, uint16_t* revn,
                                  int* has_n, cudaStream_t st) {
    const long long nw = (n + 15) / 16;
    if (nw == 0) return cudaSuccess;
    k_reverse_packed<<<(unsigned)((nw + 255) / 256), 256, 0, st>>>(fwd, fwdn, n, rev, revn, has_n);
    return cudaGetLastError();
}

// Inspector order (LPT before the inspector; the paper notes the inspector cannot know lengths): a cheap
// predictor per side and a radix sort of the sides by it, longest first, so long homologous extensions start early
// instead of forming a tail at the end of the persistent inspector.  Only the ORDER changes: results are identical.
// Predictor: an x-drop walk along the seed's diagonal that may step over up to PREDICT_SHIFTS one-base indels
// (when the walk drops X below its best, it resumes from the best point on the better of the two neighbouring
// diagonals, judged on the next 8 bases), capped at PREDICT_CAP bases: chance seeds stop after a few bases, short
// homology at its end, long homology saturates.
constexpr int PREDICT_CAP = 2047, PREDICT_SHIFTS = 16, PREDICT_BITS = 11;
__device__ __forceinline__ int predict_score8(const DevParams& P, const uint32_t* A, long long a0, long long na,
                                              const uint32_t* B, long long b0, long long nb, long long i, long long j) {
    int sc = 0;
    for (int k = 0; k < 8 && i + k < na && j + k < nb; ++k)
        sc += P.sv[5 * base_at(B, b0 + j + k) + base_at(A, a0 + i + k)] - P.OE;
    return sc;
}
__global__ void k_predict(Batch b, DevParams P, int nsides, unsigned* keys, int* vals) {
    const int side = blockIdx.x * blockDim.x + threadIdx.x;
    if (side >= nsides) return;
    const int seed = side >> 1;
    long long tpos = b.seeds[2 * seed], qpos = b.seeds[2 * seed + 1];
    if (tpos < 0 || tpos > b.tlen || qpos < 0 || qpos > b.qlen) tpos = qpos = 0;
    const uint32_t *A, *B;
    long long a0, b0, na, nb;
    if (side & 1) {
        A = b.Tf; a0 = tpos; B = b.Qf; b0 = qpos;
        na = (long long)b.tlen - tpos; nb = (long long)b.qlen - qpos;
    } else {
        A = b.Tr; a0 = b.tlen - tpos; B = b.Qr; b0 = b.qlen - qpos;
        na = tpos; nb = qpos;
    }
    na = min(na, (long long)PREDICT_CAP);
    const int X = 4 * P.OE;  // x-drop of the walk (a few mismatches of headroom)
    int sc = 0, best = 0, shifts = 0;
    long long i = 0, j = 0, bi = 0, bj = 0;
    while (i < na && j < nb) {
        sc += P.sv[5 * base_at(B, b0 + j) + base_at(A, a0 + i)] - P.OE;
        ++i;
        ++j;
        if (sc > best) {
            best = sc;
            bi = i;
            bj = j;
        } else if (sc < best - X) {
            if (++shifts > PREDICT_SHIFTS) break;
            const int sd = predict_score8(P, A, a0, na, B, b0, nb, bi + 1, bj);  // skip a target base
            const int si = predict_score8(P, A, a0, na, B, b0, nb, bi, bj + 1);  // skip a query base
            // resume only if a neighbouring diagonal clearly continues (~6 of 8 bases matching): chance
            // seeds stop at their first drop, so the walk costs them a few dozen base reads
            const int need = 3 * (P.sv[0] - P.OE);  // 3 x sub(A, A)
            if (sd < need && si < need) break;
            i = sd >= si ? bi + 1 : bi;
            j = sd >= si ? bj : bj + 1;
            sc = best - P.OE;
        }
    }
    keys[side] = (unsigned)(bi < PREDICT_CAP ? bi : PREDICT_CAP);
    vals[side] = side;
}

size_t order_tmp_bytes(int n) {
    size_t bytes = 0;
    cub::DeviceRadixSort::SortPairsDescending(nullptr, bytes, (const unsigned*)nullptr, (unsigned*)nullptr,
                                              (const int*)nullptr, (int*)nullptr, n > 0 ? n : 1);
    return bytes;
}

cudaError_t launch_order(const Batch& b, const DevParams& P, int nsides, unsigned* keys_in, unsigned* keys_out,
                         int* vals_in, int* order, void* tmp, size_t tmp_bytes, cudaStream_t st) {
    if (nsides == 0) return cudaSuccess;
    k_predict<<<(nsides + 255) / 256, 256, 0, st>>>(b, P, nsides, keys_in, vals_in);
    size_t bt = tmp_bytes;
    return cub::DeviceRadixSort::SortPairsDescending(tmp, bt, keys_in, keys_out, vals_in, order, nsides, 0,
                                                     PREDICT_BITS, st);
}

__global__ void k_validate_seeds(const long long* __restrict__ seeds, int n, int tlen, int qlen, long long* bad) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) return;
    const long long t = seeds[2 * s], q = seeds[2 * s + 1];
    if (t < 0 || t > tlen || q < 0 || q > qlen) atomicMin(bad, (long long)s);
}

cudaError_t launch_validate_seeds(const long long* seeds, int n, int tlen, int qlen, long long* bad,
                                  cudaStream_t st) {
    if (n == 0) return cudaSuccess;
    k_validate_seeds<<<(n + 255) / 256, 256, 0, st>>>(seeds, n, tlen, qlen, bad);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------- sides
// Side 2s is seed s's left extension (A_k = T[tpos-k], B_k = Q[qpos-k]: reversed copies starting at
// tlen - tpos, qlen - qpos), side 2s+1 its right extension (A_k = T[tpos+k-1], B_k = Q[qpos+k-1]) -- P:168.
template <bool NM>
__device__ __forceinline__ void setup_side(const Batch& b, int side, SideIO& io) {
    const int seed = side >> 1;
    long long tpos = b.seeds[2 * seed], qpos = b.seeds[2 * seed + 1];
    // a seed outside [0, len] is reported by k_validate_seeds (FASTZ_ERANGE, the batch's results are void);
    // until the host sees that flag its sides run as empty extensions at the origin, so no kernel ever reads
    // outside the sequences
    if (tpos < 0 || tpos > b.tlen || qpos < 0 || qpos > b.qlen) tpos = qpos = 0;
    if (side & 1) {
        io.Apk = b.Tf; io.Aoff = tpos; io.M = (int)(b.tlen - tpos);
        io.Bpk = b.Qf; io.Boff = qpos; io.Bmax = (int)(b.qlen - qpos);
    } else {
        io.Apk = b.Tr; io.Aoff = b.tlen - tpos; io.M = (int)tpos;
        io.Bpk = b.Qr; io.Boff = b.qlen - qpos; io.Bmax = (int)qpos;
    }
    if constexpr (NM) {
        __syncwarp();  // the previous side's last mask reads are done
        io.ws->anm = (side & 1) ? b.TfN : b.TrN;
        io.ws->bnm = (side & 1) ? b.QfN : b.QrN;
        __syncwarp();
    }
    io.N = io.Bmax;
}

constexpr int OP_M = 0, OP_I = 1, OP_D = 2;

// the substitution table is sized for the batch's alphabet: the N-free layout (10 KB) leaves 9 KB more of the SM's
// unified memory to L1 than the N-aware one
template <bool NM>
struct SmemDP {
    alignas(16) int subtab[SubTab<NM>::INTS];
    WarpSmem w[WARPS];
    uint8_t ecodes[WARPS][EAGER_W * EAGER_W + 15];
};

template <bool NM>
__device__ __forceinline__ void smem_init(SmemDP<NM>& sm, const DevParams& P) {
    using T = SubTab<NM>;
    for (int idx = threadIdx.x; idx < T::INTS / 2; idx += blockDim.x) {
        const int e = idx / SUBTAB_REP, code = e / (T::NB * T::NB), a0 = (e / T::NB) % T::NB, a1 = e % T::NB;
        sm.subtab[2 * idx] = P.sv[5 * code + a0];
        sm.subtab[2 * idx + 1] = P.sv[5 * code + a1];
    }
    // the column-code ring is read ahead of the strip's first column during ramp-up (dead cells): it must
    // always hold valid table offsets
    for (int idx = threadIdx.x; idx < WARPS * (CP_RING + BLK); idx += blockDim.x)
        sm.w[idx / (CP_RING + BLK)].co[idx % (CP_RING + BLK)] = 4 * T::CODE;
    __syncthreads();
}

template <bool NM>
__device__ __forceinline__ void io_init(SideIO& io, SmemDP<NM>& sm, int4* ring, int rmask, int warp_slot, int warp) {
    io.ring = ring + (size_t)warp_slot * (size_t)(rmask + 1);
    io.rmask = rmask;
    io.ws = &sm.w[warp];
    io.subtab = (unsigned)__cvta_generic_to_shared(sm.subtab);
    io.ecodes = sm.ecodes[warp];
    io.eager_max = -1;
    io.codes = nullptr;
    io.stab = nullptr;
    io.budget = INT_MAX;
    io.ps = nullptr;
    io.wi = warp;
    io.K = WARPS;
    io.maxsw = 0;
    io.wlim = 0;
    io.xexp = 0;
}

// eager traceback by lane 0 over the 17x17 corner codes; returns ops (2 bits each, peak -> origin)
__device__ __forceinline__ unsigned long long eager_walk(const uint8_t* ec, int i, int j, int& nops) {
    unsigned long long ops = 0;
    nops = 0;
    int state = 0;
    while (i > 0 || j > 0) {
        const uint32_t code = ec[i * EAGER_W + j];
        if (state == 0) {
            const uint32_t src = code & 3u;
            if (src == 0) {
                ops |= (unsigned long long)OP_M << (2 * nops);
                ++nops; --i; --j;
                continue;
            }
            state = (int)src;
        }
        if (state == 1) {
            ops |= (unsigned long long)OP_D << (2 * nops);
            ++nops;
            state = (code >> 2) & 1u ? 1 : 0;
            --i;
        } else {
            ops |= (unsigned long long)OP_I << (2 * nops);
            ++nops;
            state = (code >> 3) & 1u ? 2 : 0;
            --j;
        }
    }
    return ops;
}

__device__ __forceinline__ void write_side(const DevParams& P, const SideArrays& sa, int side, const SideOut& o,
                                           uint32_t flags, unsigned long long ops, int nops) {
    sa.score[side] = o.best + P.OE;
    sa.ti[side] = o.bi;
    sa.qj[side] = o.bj;
    sa.flags[side] = flags | ((uint32_t)nops << 8);
    sa.eops[side] = ops;
    const bool notrim = P.options & OPT_NO_TRIM;  // executor redoes every explored strip (ablation, P:172 off)
    sa.bound[side] = (flags & SF_EAGER) ? 0 : (notrim ? o.words : o.bound_words);
    sa.maxsw[side] = (flags & SF_EAGER) ? 0 : (notrim ? o.maxsw_all : o.bound_maxsw);
    sa.nstrip[side] = notrim ? o.nstrips : -1;
}

// register budget of the inspector: 72 registers = 7 resident CTAs of 4 warps per SM measured fastest.  ptxas's
// own choice is fragile (72 or 115-122 registers for near-identical code, the latter at 4 CTAs per SM and ~20%
// slower): the N-free instantiation lands at 72 by itself (an explicit cap there costs 3 instructions per step),
// the N-aware one (k_inspect_n) is capped with __maxnreg__ (any explicit attribute on the N-free kernel, even
// __maxnreg__(255) or a minimum of 1 CTA, moves it to ~120 registers).
// ------------------------------------------------------------------------------------------------- inspector
// Persistent: each warp pops one-sided extensions from an atomic queue (load balance replaces the paper's
// 32 CUDA streams).  Score-only DP + eager 17x17 corner codes; when the peak lies inside the
// eager window the warp's lane 0 walks the codes at once and the side skips the executor.
// A side still running after `budget` strips is handed to the block-per-side inspector (escalation).
template <int R, bool NM>
__device__ __forceinline__ void inspect_body(const DevParams& P, const Batch& b, int4* ring, int rmask,
                                             const SideArrays& sa, const ExecPlan& pl, int budget,
                                             const int* __restrict__ slist, int nlist) {
    __shared__ SmemDP<NM> sm;
    smem_init<NM>(sm, P);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    SideIO io;
    io_init(io, sm, ring, rmask, blockIdx.x * WARPS + warp, warp);
    io.eager_max = P.eager_max;
    io.budget = budget;
    // slist: the order in which to take the sides (predicted-longest first), or the sides whose band overflowed
    // the regular ring, re-inspected with the wide ring (k_mark_wide flags them afterwards)
    const int nsides = slist ? nlist : 2 * b.nseeds;
    for (;;) {
        int side = 0;
        if (lane == 0) side = atomicAdd(&pl.counters[0], 1);
        side = __shfl_sync(FULL, side, 0);
        if (side >= nsides) break;
        if (slist) side = slist[side];
        setup_side<NM>(b, side, io);
        SideOut o;
        run_side<R, MODE_INSPECT, true, false, NM>(P, io, o);
        __syncwarp();  // eager corner codes (shared memory) written by lanes 0..4 -> read by lane 0
        if (lane == 0) {
            if (o.flags & SF_ESCALATE) {
                pl.esc[atomicAdd(&pl.counters[21], 1)] = side;
            } else {
                uint32_t flags = o.flags;
                unsigned long long ops = 0;
                int nops = 0;
                if (o.bi <= P.eager_max && o.bj <= P.eager_max && !(flags & (SF_RING | SF_OVERFLOW)) &&
                    !(P.options & OPT_NO_EAGER)) {
                    ops = eager_walk(io.ecodes, o.bi, o.bj, nops);
                    flags |= SF_EAGER;
                }
                write_side(P, sa, side, o, flags, ops, nops);
            }
        }
        __syncwarp();
    }
}

#ifndef INSPECT_ATTR
#define INSPECT_ATTR __launch_bounds__(WARPS * 32)
#endif
template <int R>
__global__ void INSPECT_ATTR k_inspect(DevParams P, Batch b, int4* ring, int rmask, SideArrays sa,
                                                         ExecPlan pl, int budget, const int* slist, int nlist) {
    inspect_body<R, false>(P, b, ring, rmask, sa, pl, budget, slist, nlist);
}
template <int R>
#ifndef INSPECT_N_MAXREG
#define INSPECT_N_MAXREG 80  // 6 CTAs per SM: measured 2% faster than 72 (which spills) on C2 with N runs
#endif
__global__ void __maxnreg__(INSPECT_N_MAXREG) k_inspect_n(DevParams P, Batch b, int4* ring, int rmask,
                                                                           SideArrays sa, ExecPlan pl, int budget,
                                                                           const int* slist, int nlist) {
    inspect_body<R, true>(P, b, ring, rmask, sa, pl, budget, slist, nlist);
}

// ------------------------------------------------------------------------------------------- packed inspector
}  // namespace fz
#include "pair.cuh"
namespace fz {
// One persistent launch for the whole inspection when the packed inspector is on (no tails between phases):
//   phase 1: the predicted-long sides order[0, nlong) one per warp in the 32-bit inspector (inline eager walk);
//   phase 2: the other sides two per warp in the packed inspector (queue counters[32]);
//   then the sides phase 2 abandoned (value cap, or too many strips: pl.redo, pre-set to -1, counters[30] pushes,
//   counters[34] claims), in the 32-bit inspector, by whichever warp claims them first (see below).
// The 32-bit path reads the packed inspector's table (the same layout as dp.cuh's SubTab<false>).
struct SmemMixed {
    alignas(16) int subtab[PSUB_INTS];
    union Warp {
        WarpSmem w32;
        PairWarp wp;
    } w[WARPS];
    uint8_t ecodes[WARPS][EAGER_W * EAGER_W + 15];
};

// 72 registers = 7 CTAs per SM; ptxas's own choice for the fused code is 122 (4 CTAs).  At 72 the 32-bit steady loop
// runs 57.0 instructions per step (55.4 in k_inspect) and the packed loop 88.6, no spills in
// either loop (SASS, tools/sass_fastpath.py).
#ifndef MIXED_MAXREG
#define MIXED_MAXREG 72
#endif
template <int R>
__device__ __forceinline__ void inspect_one32(const DevParams& P, const Batch& b, const SideArrays& sa,
                                              const ExecPlan& pl, SideIO& io, int side, int budget) {
    const int lane = threadIdx.x & 31;
    __syncwarp();
    // (re)enter 32-bit mode: the union's column-code ring must hold 32-bit table offsets
    for (int i = lane; i < CP_RING + BLK; i += 32) io.ws->co[i] = 4 * SubTab<false>::CODE;
    __syncwarp();
    setup_side<false>(b, side, io);
    SideOut o;
    run_side<R, MODE_INSPECT, true, false, false>(P, io, o);
    __syncwarp();
    if (lane == 0) {
        if (o.flags & SF_ESCALATE) {
            pl.esc[atomicAdd(&pl.counters[21], 1)] = side;
        } else {
            uint32_t flags = o.flags;
            unsigned long long ops = 0;
            int nops = 0;
            if (o.bi <= P.eager_max && o.bj <= P.eager_max && !(flags & (SF_RING | SF_OVERFLOW)) &&
                !(P.options & OPT_NO_EAGER)) {
                ops = eager_walk(io.ecodes, o.bi, o.bj, nops);
                flags |= SF_EAGER;
            }
            write_side(P, sa, side, o, flags, ops, nops);
        }
    }
    __syncwarp();
}

template <int R>
__global__ void __maxnreg__(MIXED_MAXREG) k_inspect_mixed(DevParams P, PairParams Q, Batch b, int4* ring,
                                                              int rmask, SideArrays sa, ExecPlan pl,
                                                              const int* order, int ns, int nlong, int n1,
                                                              int budget, long long* dbg) {
    __shared__ SmemMixed sm;
    // order[0, nlong): the predicted-long head of the order; the first n1 of them (n1 = nlong, or 0 when a
    // concurrent k_inspect takes them) run here in phase 1 (queue counters[35]); order[nlong, ns) are packed
    for (int idx = threadIdx.x; idx < PSUB_INTS / 2; idx += blockDim.x) {
        const int e = idx / SUBTAB_REP, code = e / 16, a0 = (e / 4) % 4, a1 = e % 4;
        sm.subtab[2 * idx] = P.sv[5 * code + a0];
        sm.subtab[2 * idx + 1] = P.sv[5 * code + a1];
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int slot = blockIdx.x * WARPS + warp;
    const unsigned subtab = (unsigned)__cvta_generic_to_shared(sm.subtab);
    SideIO io;
    io.ring = ring + (size_t)slot * (size_t)(rmask + 1);
    io.rmask = rmask;
    io.ws = &sm.w[warp].w32;
    io.subtab = subtab;
    io.ecodes = sm.ecodes[warp];
    io.eager_max = P.eager_max;
    io.codes = nullptr;
    io.stab = nullptr;
    io.budget = budget;
    io.ps = nullptr;
    io.wi = warp;
    io.K = WARPS;
    io.maxsw = 0;
    io.wlim = 0;
    io.xexp = 0;
    __shared__ int owns[WARPS];  // redo side claimed by the warp (index into pl.redo), -1: none
    if (lane == 0) owns[warp] = -1;
    __syncwarp();
    volatile int* ctr = pl.counters;
    volatile int* redo = pl.redo;
    // claim a pushed redo side (lane 0): index or -1
    auto claim = [&]() -> int {
        int c = ctr[34];
        while (c < ctr[30]) {
            const int o = atomicCAS(&pl.counters[34], c, c + 1);
            if (o == c) return c;
            c = o;
        }
        return -1;
    };
    // One loop, one 32-bit call site (each inlined copy of the 32-bit inspector costs registers and instructions).
    // phase 1: predicted-long sides (claimed redo sides first, should any appear); phase 2: packed sides -- a warp
    // that claims a redo side stops taking packed sides, runs it in 32 bits once both halves are idle, then returns
    // to the packed queue.  No warp needs to wait for late redo sides: a side is pushed in finish() and the pusher's
    // very next pop() claims any unclaimed push, so every pushed side has a live claimer; a warp leaves when its
    // pops find the packed queue empty and nothing left to claim.
    int phase = 1;
    long long tph[4] = {clock64(), 0, 0, 0};  // diagnostics: clock at start, end of phase 1, end of phase 2
    int n32 = 0;
    for (;;) {
        int side = -1, c = -1;
        bool exhausted = false;
        if (phase == 2) {
            exhausted = run_pairs<R>(P, Q, b, reinterpret_cast<int2*>(io.ring), rmask, sa, pl, &sm.w[warp].wp,
                                     subtab, order ? order + nlong : nullptr, ns - nlong, &pl.counters[32], dbg,
                                     &owns[warp]);
            __syncwarp();
            c = owns[warp];
            __syncwarp();
            if (lane == 0) owns[warp] = -1;
        }
        int next = phase;
        if (lane == 0) {
            if (phase == 1) {
                c = claim();
                if (c < 0) {
                    const int item = atomicAdd(&pl.counters[35], 1);
                    if (item < n1) side = order ? order[item] : item;
                    else next = 2;
                }
            }
            if (c >= 0)
                while ((side = redo[c]) < 0) __nanosleep(100);  // the push lands right after the count
        }
        __syncwarp();  // lane 0 spun in claim / push waits: reconverge before the collectives
        side = __shfl_sync(FULL, side, 0);
        next = __shfl_sync(FULL, next, 0);
        if (next != phase) tph[phase] = clock64();
        phase = next;
        if (side >= 0) {
            inspect_one32<R>(P, b, sa, pl, io, side, phase == 1 ? budget : INT_MAX);
            ++n32;
            continue;
        }
        if (exhausted) {
            tph[2] = clock64();
            break;
        }
    }
    if (dbg && lane == 0) {
        long long* d = dbg + 4 * (long long)ns + 4 * slot;
        d[0] = tph[1] - tph[0];
        d[1] = tph[2] - tph[0];
        d[2] = clock64() - tph[0];
        d[3] = n32;
    }
}

int mixed_blocks_per_sm() {
    int n = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_inspect_mixed<4>, WARPS * 32, 0);
    return n > 0 ? n : 1;
}

cudaError_t launch_inspect_mixed(int grid, const DevParams& P, const PairParams& Q, const Batch& b, int4* ring,
                                 int rmask, const SideArrays& sa, const ExecPlan& pl, const int* order, int nsides,
                                 int nlong, int n1, int budget, long long* dbg, cudaStream_t st) {
    if (nsides == 0) return cudaSuccess;
    k_inspect_mixed<4><<<grid, WARPS * 32, 0, st>>>(P, Q, b, ring, rmask, sa, pl, order, nsides, nlong, n1, budget,
                                                    dbg);
    return cudaGetLastError();
}

__global__ void k_split(const unsigned* keys, int n, unsigned thr, int* count) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    int lo = 0, hi = n;  // keys descending: first index with key < thr
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (keys[mid] >= thr) lo = mid + 1;
        else hi = mid;
    }
    *count = lo;
}

cudaError_t launch_split(const unsigned* keys_desc, int n, unsigned thr, int* count, cudaStream_t st) {
    k_split<<<1, 32, 0, st>>>(keys_desc, n, thr, count);
    return cudaGetLastError();
}

// Eager corner codes of a packed-inspector side, recomputed by one thread over [0, i*] x [0, j*] with exactly the
// inspector's cell rule (dp.cuh; the cone rule only looks inside the rectangle, reading R3), then walked as in
// inspect_body.  Only sides whose peak lies in the 17x17 corner do any work.
__global__ void k_eager(DevParams P, Batch b, SideArrays sa, int nsides) {
    const int side = blockIdx.x * blockDim.x + threadIdx.x;
    if (side >= nsides) return;
    uint32_t fl = sa.flags[side];
    if (!(fl & SF_PAIR)) return;
    fl &= ~SF_PAIR;
    const int bi = sa.ti[side], bj = sa.qj[side];
    if (bi <= P.eager_max && bj <= P.eager_max && !(fl & (SF_RING | SF_OVERFLOW)) && !(P.options & OPT_NO_EAGER)) {
        SideIO io;
        setup_side<false>(b, side, io);
        uint8_t ec[EAGER_W * EAGER_W];
        int Xr[EAGER_W], Dr[EAGER_W], Wr[EAGER_W];  // row r - 1 (row -1: the strip-0 boundary, dead, W = NEG)
        for (int c = 0; c <= bj; ++c) {
            Xr[c] = NEG;
            Dr[c] = NEG;
            Wr[c] = NEG;
        }
        const int E = P.E, OE = P.OE, Y = P.Y;
        for (int r = 0; r <= bi; ++r) {
            const int a = (r >= 1 && r <= io.M) ? base_at(io.Apk, io.Aoff + r - 1) : 0;
            int xl = NEG, il = NEG, wl = -Y - 1;  // left of column 0 (ramp-up cells: dead, W = -(Y+1))
            int xdg = r == 0 ? -OE : NEG;          // X(r-1, -1); the origin's diagonal gives H(0,0) = 0
            for (int c = 0; c <= bj; ++c) {
                const int code = (c >= 1 && c <= io.N) ? base_at(io.Bpk, io.Boff + c - 1) : 4;
                const int xu = Xr[c], du = Dr[c], wu = Wr[c];
                const int h = xdg + P.sv[5 * code + a];
                const int d = imax(du - E, xu);
                const int iv = imax(il - E, xl);
                const int sr = imax(imax(h, d), iv);
                const int thr = imax(wu, wl);
                const int xn = sr >= thr ? sr - OE : NEG;
                const int wn = imax(sr - Y, thr);
                ec[r * EAGER_W + c] = (uint8_t)cell_code(h, d, iv, du, xu, il, xl, E);
                xdg = xu;
                Xr[c] = xn;
                Dr[c] = d;
                Wr[c] = wn;
                xl = xn;
                il = iv;
                wl = wn;
            }
        }
        int nops = 0;
        const unsigned long long ops = eager_walk(ec, bi, bj, nops);
        fl |= SF_EAGER | ((uint32_t)nops << 8);
        sa.eops[side] = ops;
        sa.bound[side] = 0;
        sa.maxsw[side] = 0;
    }
    sa.flags[side] = fl;
}

cudaError_t launch_eager(const DevParams& P, const Batch& b, const SideArrays& sa, int nsides, cudaStream_t st) {
    if (nsides == 0) return cudaSuccess;
    k_eager<<<(nsides + 127) / 128, 128, 0, st>>>(P, b, sa, nsides);
    return cudaGetLastError();
}

// Block per side (long sides, escalated by k_inspect): the CTA's warps pipeline the side's strips.
template <int R, bool NM>
__global__ void __launch_bounds__(WARPS * 32) k_inspect_block(DevParams P, Batch b, int4* ring, int rmask,
                                                               SideArrays sa, ExecPlan pl) {
    __shared__ SmemDP<NM> sm;
    __shared__ PipeShared ps;
    __shared__ int cur;
    smem_init<NM>(sm, P);
    const int warp = threadIdx.x >> 5;
    for (;;) {
        if (threadIdx.x == 0) {
            const int i = atomicAdd(&pl.counters[22], 1);
            cur = i < pl.counters[21] ? pl.esc[i] : -1;
            pipe_reset(&ps);
        }
        __syncthreads();
        const int side = cur;
        if (side < 0) break;
        SideIO io;
        io_init(io, sm, ring, rmask, blockIdx.x * WARPS, warp);
        io.ps = &ps;
        setup_side<NM>(b, side, io);
        SideOut o;
        run_side<R, MODE_INSPECT, false, true, NM>(P, io, o);
        if (threadIdx.x == 0) write_side(P, sa, side, o, o.flags, 0ull, 0);
        __syncthreads();
    }
}

template <int R, bool NM>
__global__ void __launch_bounds__(WARPS * 32) k_census(DevParams P, Batch b, int4* ring, int rmask,
                                                        long long* cells, int* counter, const int* slist, int nlist) {
    __shared__ SmemDP<NM> sm;
    smem_init<NM>(sm, P);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    SideIO io;
    io_init(io, sm, ring, rmask, blockIdx.x * WARPS + warp, warp);
    const int nsides = slist ? nlist : 2 * b.nseeds;
    for (;;) {
        int side = 0;
        if (lane == 0) side = atomicAdd(counter, 1);
        side = __shfl_sync(FULL, side, 0);
        if (side >= nsides) break;
        if (slist) side = slist[side];
        setup_side<NM>(b, side, io);
        SideOut o;
        run_side<R, MODE_CENSUS, false, false, NM>(P, io, o);
        if (lane == 0) cells[side] = (o.flags & SF_RING) ? -1 : o.cells;
        __syncwarp();
    }
}

// ------------------------------------------------------------------------------------------------- executor
// Trimmed executor: the DP over [0,i*]x[0,j*] only, writing traceback codes.  Length binning
// as a schedule: the CTAs first take the long sides (bins >= 3, block per side, strips pipelined
// across the CTA's warps), then every warp takes short sides (bins 1-2, warp per side), larger bins first.
// ptxas's natural 96 registers (5 CTAs per SM).  Capped at 80 (6 CTAs, -DEXECUTE_MIN_BLOCKS=6) the warp-per-side
// loop keeps its instruction count (SASS 95 vs 94.5 per 4-cell step) but the block-per-side loop grows (111 vs
// 103) and every config measured slower (tools/config_sweep.py: C2 12.0 vs 10.9 ms, C3 152.7 vs 148.0 ms, C1 124.3
// vs 120.5 ms; profiles/r2/configs_sweep.jsonl)
#ifdef EXECUTE_MIN_BLOCKS
#define EXECUTE_ATTR __launch_bounds__(WARPS * 32, EXECUTE_MIN_BLOCKS)
#else
#define EXECUTE_ATTR __launch_bounds__(WARPS * 32)
#endif
template <int R, bool NM>
__global__ void EXECUTE_ATTR k_execute(DevParams P, Batch b, int4* ring, int rmask,
                                                         SideArrays sa, ExecPlan pl, int lo, int hi, int nblock,
                                                         long long base, Outputs out, int wide) {
    // wide = 1: this launch (the wide ring) runs only the SF_WIDE sides of the range, wide = 0 all others
    __shared__ SmemDP<NM> sm;
    __shared__ PipeShared ps;
    __shared__ int cur;
    smem_init<NM>(sm, P);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned long long written = 0;  // code words written by this thread's sides (stats; one atomic at the end)
    for (;;) {  // block phase
        if (threadIdx.x == 0) {
            const int i = lo + atomicAdd(&pl.counters[23], 1);
            cur = i < (hi < nblock ? hi : nblock) ? pl.list[i] : -1;
            pipe_reset(&ps);
        }
        __syncthreads();
        const int side = cur;
        if (side < 0) break;
        if (((sa.flags[side] & SF_WIDE) != 0) != (wide != 0)) {
            __syncthreads();  // cur is rewritten by thread 0 next iteration
            continue;
        }
        SideIO io;
        io_init(io, sm, ring, rmask, blockIdx.x * WARPS, warp);
        io.ps = &ps;
        setup_side<NM>(b, side, io);
        if (!(P.options & OPT_NO_TRIM)) {  // trimmed executor: the rectangle up to the peak
            io.M = sa.ti[side];
            io.N = sa.qj[side];
        }
        io.codes = out.codes + (pl.woff[side] - base);
        io.stab = out.stab + pl.soff[side];
        io.maxsw = sa.maxsw[side];
        io.xexp = (P.options & OPT_NO_TRIM) ? INT_MIN : sa.score[side] - P.OE + ((P.options & OPT_SELFCHECK_TEST) ? 1 : 0);
        SideOut o;
        run_side<R, MODE_EXEC, false, true, NM>(P, io, o);
        if (threadIdx.x == 0 && (o.flags & SF_RING)) atomicOr(&sa.flags[side], SF_RING);
        if (threadIdx.x == 0 && o.checkfail) atomicAdd(&pl.counters[26], 1);
        if (threadIdx.x == 0) written += (unsigned long long)o.words;
        __syncthreads();
    }
    SideIO io;
    io_init(io, sm, ring, rmask, blockIdx.x * WARPS + warp, warp);
    for (;;) {  // warp phase
        int idx = 0;
        if (lane == 0) idx = (lo > nblock ? lo : nblock) + atomicAdd(&pl.counters[1], 1);
        idx = __shfl_sync(FULL, idx, 0);
        if (idx >= hi) break;
        const int side = pl.list[idx];
        if (((sa.flags[side] & SF_WIDE) != 0) != (wide != 0)) continue;
        setup_side<NM>(b, side, io);
        if (!(P.options & OPT_NO_TRIM)) {
            io.M = sa.ti[side];
            io.N = sa.qj[side];
        }
        io.codes = out.codes + (pl.woff[side] - base);
        io.stab = out.stab + pl.soff[side];
        io.wlim = sa.bound[side];
        io.xexp = (P.options & OPT_NO_TRIM) ? INT_MIN : sa.score[side] - P.OE + ((P.options & OPT_SELFCHECK_TEST) ? 1 : 0);
        SideOut o;
        run_side<R, MODE_EXEC, false, false, NM>(P, io, o);
        if (lane == 0 && (o.flags & SF_RING)) atomicOr(&sa.flags[side], SF_RING);
        if (lane == 0 && o.checkfail) atomicAdd(&pl.counters[26], 1);
        if (lane == 0) written += (unsigned long long)o.words;
        __syncwarp();
    }
    if (lane == 0 && written) atomicAdd((unsigned long long*)(pl.totals + 6), written);
}

// ------------------------------------------------------------------------------------------------- traceback
// One thread per executed side (inter-seed traceback parallelism).  Walks the 4-bit codes from
// (i*, j*) in state S to the origin; emits run-length ops (len << 2 | op) in peak -> origin order.
#ifndef TB_PREFETCH
#define TB_PREFETCH 32
#endif
template <int R>
__global__ void k_traceback(SideArrays sa, ExecPlan pl, int lo, int hi, long long base, Outputs out) {
    constexpr int H = 32 * R, SPW = 8 / R;
    const int idx = lo + blockIdx.x * blockDim.x + threadIdx.x;
    if (idx >= hi) return;
    const int side = pl.list[idx];
    const uint32_t* __restrict__ codes = out.codes + (pl.woff[side] - base);
    const int2* __restrict__ stab = out.stab + pl.soff[side];
    uint32_t* __restrict__ runs = out.runs + pl.roff[side];
    int i = sa.ti[side], j = sa.qj[side], state = 0, nr = 0;
    uint32_t cur = 0xffffffffu, len = 0;
    auto emit = [&](uint32_t op) {
        if (op == cur) {
            ++len;
        } else {
            if (len) runs[nr++] = (len << 2) | cur;
            cur = op;
            len = 1;
        }
    };
    // the walk is a chain of dependent loads: cache the strip entry and the current code word, and prefetch
    // the word a few diagonal steps ahead (the common direction) into L1
    int scur = -1;
    int2 st = make_int2(0, 0);
    long long wcur = -1;
    uint32_t w = 0;
    while (i > 0 || j > 0) {
        const int s = i / H, lr = i - s * H, ln = lr / R, k = lr - ln * R;
        if (s != scur) {
            st = stab[s];
            scur = s;
        }
        const int t = j - st.x + ln;
        const long long wi = (long long)st.y + (long long)(t / SPW) * 32 + ln;
        if (wi != wcur) {
            w = codes[wi];
            wcur = wi;
            // ~HBM latency / (cycles per step): 32 diagonal steps = 16 lines ahead, within this strip
            const int i2 = i - TB_PREFETCH, j2 = j - TB_PREFETCH;
            if (i2 >= s * H && j2 >= st.x) {
                const int l2 = (i2 - s * H) / R;
                const long long w2 = (long long)st.y + (long long)((j2 - st.x + l2) / SPW) * 32 + l2;
                asm volatile("prefetch.global.L2 [%0];" ::"l"(codes + w2));
            }
        }
        const uint32_t code = (w >> ((((t % SPW) * R) + k) * 4)) & 15u;
        // branch-free step (the 32 walks of a warp diverge otherwise): in state S the cell's source decides
        // (H -> M, D -> enter D, I -> enter I; executor code: bit 1 = I, else bit 0 = D), in a gap state the
        // move is the gap's; one op per iteration
        const int eff = state == 0 ? ((code & 2u) ? 2 : (int)(code & 1u)) : state;  // 0 M, 1 D, 2 I
        const uint32_t op = eff == 0 ? (uint32_t)OP_M : (eff == 1 ? (uint32_t)OP_D : (uint32_t)OP_I);
        const bool ext = eff == 1 ? ((code >> 2) & 1u) : ((code >> 3) & 1u);
        state = eff == 0 ? 0 : (ext ? eff : 0);
        i -= eff != 2;
        j -= eff != 1;
        emit(op);
    }
    if (len) runs[nr++] = (len << 2) | cur;
    out.nruns[side] = nr;
}

// Warp per side (long sides, list positions < nblock = bins >= 3): the walk is the same chain of dependent
// steps, but the code words come from a shared-memory window that the warp refills with coalesced loads (64
// word rows = 8 KB per warp: the next 64 * SPW steps to the left of the current one in the strip), so a
// step costs a shared-memory read instead of an HBM round trip.  All 32 lanes walk in lockstep (uniform control
// flow); lane 0 writes the runs.
constexpr int TBW_ROWS = 64;  // word rows (32 words each) per window
template <int R>
__global__ void __launch_bounds__(128) k_traceback_warp(SideArrays sa, ExecPlan pl, int lo, int hi, long long base,
                                                        Outputs out) {
    constexpr int H = 32 * R, SPW = 8 / R;
    __shared__ uint32_t win[4][TBW_ROWS * 32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int idx = lo + blockIdx.x * 4 + warp;
    if (idx >= hi) return;
    uint32_t* wbuf = win[warp];
    const int side = pl.list[idx];
    const uint32_t* __restrict__ codes = out.codes + (pl.woff[side] - base);
    const int2* __restrict__ stab = out.stab + pl.soff[side];
    uint32_t* __restrict__ runs = out.runs + pl.roff[side];
    int i = sa.ti[side], j = sa.qj[side], state = 0, nr = 0;
    uint32_t cur = 0xffffffffu, len = 0;
    auto emit = [&](uint32_t op) {
        if (op == cur) {
            ++len;
        } else {
            if (len && lane == 0) runs[nr] = (len << 2) | cur;
            nr += len ? 1 : 0;
            cur = op;
            len = 1;
        }
    };
    int scur = -1, rlo = 0, rhi = 0;  // window = word rows [rlo, rhi) of strip scur
    int2 st = make_int2(0, 0);
    while (i > 0 || j > 0) {
        const int s = i / H, lr = i - s * H, ln = lr / R, k = lr - ln * R;
        if (s != scur) {
            st = stab[s];
            scur = s;
            rhi = 0;
            rlo = 1;  // empty
        }
        const int t = j - st.x + ln;
        const int wr = t / SPW;
        if (wr < rlo || wr >= rhi) {  // refill: rows [wr - TBW_ROWS + 1, wr] (the walk moves to smaller t)
            rhi = wr + 1;
            rlo = rhi - TBW_ROWS > 0 ? rhi - TBW_ROWS : 0;
            __syncwarp();
            // the window is one contiguous, 128-byte aligned run of (rhi - rlo) * 32 words: 16-byte cp.async
            // chunks, all in flight at once (one memory latency per refill instead of one per row batch)
            const uint32_t* src = codes + (long long)st.y + (long long)rlo * 32;
            const unsigned dst = (unsigned)__cvta_generic_to_shared(wbuf);
            const int nw = (rhi - rlo) * 32;
            for (int c = lane * 4; c < nw; c += 128)
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + 4u * (unsigned)c), "l"(src + c)
                             : "memory");
            asm volatile("cp.async.wait_all;" ::: "memory");
            __syncwarp();
        }
        const uint32_t w = wbuf[(wr - rlo) * 32 + ln];
        const uint32_t code = (w >> ((((t % SPW) * R) + k) * 4)) & 15u;
        const int eff = state == 0 ? ((code & 2u) ? 2 : (int)(code & 1u)) : state;  // 0 M, 1 D, 2 I
        const uint32_t op = eff == 0 ? (uint32_t)OP_M : (eff == 1 ? (uint32_t)OP_D : (uint32_t)OP_I);
        const bool ext = eff == 1 ? ((code >> 2) & 1u) : ((code >> 3) & 1u);
        state = eff == 0 ? 0 : (ext ? eff : 0);
        i -= eff != 2;
        j -= eff != 1;
        emit(op);
    }
    if (len) {
        if (lane == 0) runs[nr] = (len << 2) | cur;
        ++nr;
    }
    if (lane == 0) out.nruns[side] = nr;
}

// ------------------------------------------------------------------------------------------------- binning
// Bins by max(i*, j*) (512, 2048, 8192, 32768, then 4x): bin 0 = eager.
__device__ __forceinline__ int bin_of(int m) {
    if (m <= 512) return 1;
    if (m <= 2048) return 2;
    if (m <= 8192) return 3;
    if (m <= 32768) return 4;
    if (m <= 131072) return 5;
    return 6;
}

template <int R>
__global__ void k_bin_count(DevParams P, SideArrays sa, int nsides, ExecPlan pl, long long* words, long long* strips,
                            long long* runs, int bblock) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= nsides) return;
    uint32_t fl = sa.flags[s];
    if ((P.options & OPT_TB_ABOVE_K) && sa.score[s & ~1] + sa.score[s | 1] < P.K) {
        fl |= SF_NOTB;  // NEXT-3: no traceback below the gapped threshold
        sa.flags[s] = fl;
    }
    const bool skip = fl & (SF_EAGER | SF_NOTB);
    const int ti = sa.ti[s], qj = sa.qj[s];
    int bin = skip ? 0 : bin_of(ti > qj ? ti : qj);
    if (!skip && (P.options & OPT_NO_BINNING)) bin = 1;  // one queue, warp per side (ablation)
    pl.bin[s] = bin;
    atomicAdd(&pl.counters[2 + bin], 1);
    if (fl & SF_RING) {  // band wider than the ring: re-inspected with a wider ring (api.cu)
        atomicOr(&pl.counters[20], 1);
        pl.wide[atomicAdd(&pl.counters[24], 1)] = s;
    }
    const long long ns = sa.nstrip[s] >= 0 ? sa.nstrip[s] : ti / (32 * R) + 1;
    // bins >= bblock run block per side: strip s of the side owns words [s * maxsw, (s + 1) * maxsw)
    words[s] = skip ? 0 : (bin >= bblock ? ns * (long long)sa.maxsw[s] : sa.bound[s]);
    strips[s] = skip ? 0 : ns;
    runs[s] = skip ? 0 : (long long)ti + qj + 1;
}

__global__ void k_bin_offsets(ExecPlan pl, int nsides, const long long* words, const long long* strips,
                              const long long* runs, int bblock) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    int run = 0, nblock = 0;
    for (int bin = 6; bin >= 1; --bin) {  // larger bins first
        pl.counters[10 + bin] = run;
        run += pl.counters[2 + bin];
        if (bin == bblock) nblock = run;
    }
    if (nsides > 0) {
        pl.totals[1] = pl.soff[nsides - 1] + strips[nsides - 1];
        pl.totals[2] = pl.roff[nsides - 1] + runs[nsides - 1];
    } else {
        pl.totals[0] = pl.totals[1] = pl.totals[2] = 0;
    }
    pl.totals[3] = run;
    pl.totals[4] = nblock;
}

// pool offsets in executor (list) order, so that a wave is a contiguous range of the list
__global__ void k_list_words(ExecPlan pl, const long long* words, long long* wl, int nsides) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    // positions past the executor list are scanned too (the scan runs over nsides): define them as 0
    if (i < nsides) wl[i] = i < (int)pl.totals[3] ? words[pl.list[i]] : 0;
}
__global__ void k_list_offsets(ExecPlan pl, const long long* wlo, const long long* wl) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const int n = (int)pl.totals[3];
    if (i < n) pl.woff[pl.list[i]] = wlo[i];
    if (i == 0) pl.totals[0] = n > 0 ? wlo[n - 1] + wl[n - 1] : 0;
}

__global__ void k_bin_scatter(ExecPlan pl, int nsides) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= nsides) return;
    const int bin = pl.bin[s];
    if (bin == 0) return;
    const int pos = atomicAdd(&pl.counters[10 + bin], 1);
    pl.list[pos] = s;
}

__global__ void k_mark_wide(SideArrays sa, const int* list, int n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) sa.flags[list[i]] |= SF_WIDE;
}

cudaError_t launch_mark_wide(const SideArrays& sa, const int* list, int n, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    k_mark_wide<<<(n + 255) / 256, 256, 0, st>>>(sa, list, n);
    return cudaGetLastError();
}

__global__ void k_wide_list(SideArrays sa, int nsides, int* list, int* count) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s < nsides && (sa.flags[s] & SF_WIDE)) list[atomicAdd(count, 1)] = s;
}

cudaError_t launch_wide_list(const SideArrays& sa, int nsides, int* list, int* count, cudaStream_t st) {
    cudaError_t e = cudaMemsetAsync(count, 0, 4, st);
    if (e != cudaSuccess || nsides == 0) return e;
    k_wide_list<<<(nsides + 255) / 256, 256, 0, st>>>(sa, nsides, list, count);
    return cudaGetLastError();
}

// LPT order inside the block-per-side bins (long problems first): list[0, nblock) sorted by descending
// executor words (proportional to the trimmed cells), then the pool offsets are recomputed in the new list order.
__global__ void k_lpt_keys(ExecPlan pl, const long long* words, int nblock, long long* keys, int* vals) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < nblock) {
        const int side = pl.list[i];
        keys[i] = words[side];
        vals[i] = side;
    }
}

size_t lpt_tmp_bytes(int n) {
    size_t bytes = 0;
    cub::DeviceRadixSort::SortPairsDescending(nullptr, bytes, (const long long*)nullptr, (long long*)nullptr,
                                              (const int*)nullptr, (int*)nullptr, n > 0 ? n : 1);
    return bytes;
}

cudaError_t launch_lpt(const ExecPlan& pl, int nblock, int nexec, const long long* words, long long* keys_in,
                       long long* keys_out, int* vals_in, void* sort_tmp, size_t sort_tmp_bytes, void* scan_tmp,
                       size_t scan_tmp_bytes, cudaStream_t st) {
    if (nblock < 2) return cudaSuccess;
    k_lpt_keys<<<(nblock + 255) / 256, 256, 0, st>>>(pl, words, nblock, keys_in, vals_in);
    size_t b = sort_tmp_bytes;
    cudaError_t e = cub::DeviceRadixSort::SortPairsDescending(sort_tmp, b, keys_in, keys_out, vals_in, pl.list, nblock,
                                                              0, 64, st);
    if (e != cudaSuccess) return e;
    const int g = (nexec + 255) / 256;
    k_list_words<<<g, 256, 0, st>>>(pl, words, pl.wl, nexec);
    b = scan_tmp_bytes;
    if ((e = cub::DeviceScan::ExclusiveSum(scan_tmp, b, pl.wl, pl.wlo, nexec, st)) != cudaSuccess) return e;
    k_list_offsets<<<g, 256, 0, st>>>(pl, pl.wlo, pl.wl);
    return cudaGetLastError();
}

int block_bin() {  // smallest executor bin run block per side (FASTZ_BLOCK_BIN, default 3: > 2048)
    const char* e = getenv("FASTZ_BLOCK_BIN");
    int v = e ? atoi(e) : 3;
    return v < 1 ? 1 : (v > 7 ? 7 : v);
}

size_t scan_tmp_bytes(int n) {
    size_t bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, bytes, (const long long*)nullptr, (long long*)nullptr, n > 0 ? n : 1);
    return bytes;
}

cudaError_t launch_bin(int R, const DevParams& P, const SideArrays& sa, int nsides, const ExecPlan& pl, void* tmp,
                       size_t tmp_bytes, long long* words, long long* strips, long long* runs, cudaStream_t st) {
    const int bb = (P.options & (OPT_NO_BLOCK | OPT_NO_BINNING)) ? 7 : block_bin();
    cudaError_t e;
    if (nsides > 0) {
        const int g = (nsides + 255) / 256;
        if (R == 2) k_bin_count<2><<<g, 256, 0, st>>>(P, sa, nsides, pl, words, strips, runs, bb);
        else k_bin_count<4><<<g, 256, 0, st>>>(P, sa, nsides, pl, words, strips, runs, bb);
        size_t b = tmp_bytes;
        if ((e = cub::DeviceScan::ExclusiveSum(tmp, b, strips, pl.soff, nsides, st)) != cudaSuccess) return e;
        b = tmp_bytes;
        if ((e = cub::DeviceScan::ExclusiveSum(tmp, b, runs, pl.roff, nsides, st)) != cudaSuccess) return e;
    }
    k_bin_offsets<<<1, 1, 0, st>>>(pl, nsides, words, strips, runs, bb);
    if (nsides > 0) {
        const int g = (nsides + 255) / 256;
        k_bin_scatter<<<g, 256, 0, st>>>(pl, nsides);
        long long* wl = pl.wl;
        long long* wlo = pl.wlo;
        k_list_words<<<g, 256, 0, st>>>(pl, words, wl, nsides);
        size_t b = tmp_bytes;
        if ((e = cub::DeviceScan::ExclusiveSum(tmp, b, wl, wlo, nsides, st)) != cudaSuccess) return e;
        k_list_offsets<<<g, 256, 0, st>>>(pl, wlo, wl);
    }
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------- combine
// Seed s = left side 2s (ops emitted peak -> origin in the reversed frame == forward order) followed by the
// right side 2s+1 (emitted peak -> origin == backward, so read in reverse); equal neighbours merge.
struct RunVisitor {
    const SideArrays& sa;
    const ExecPlan& pl;
    const Outputs& o;
    template <class F>
    __device__ __forceinline__ void visit(int seed, F&& f) const {
        const int L = 2 * seed, Rt = 2 * seed + 1;
        if ((sa.flags[L] | sa.flags[Rt]) & SF_NOTB) return;  // FASTZ_OPT_TRACEBACK_ABOVE_K
        uint32_t cur = 0xffffffffu;
        long long len = 0;
        auto push = [&](uint32_t op, long long n) {
            if (op == cur) {
                len += n;
            } else {
                if (len) f(cur, len);
                cur = op;
                len = n;
            }
        };
        {
            const uint32_t fl = sa.flags[L];
            if (fl & SF_EAGER) {
                const int n = (fl >> 8) & 0xff;
                const unsigned long long ops = sa.eops[L];
                for (int k = 0; k < n; ++k) push((uint32_t)(ops >> (2 * k)) & 3u, 1);
            } else {
                const uint32_t* r = o.runs + pl.roff[L];
                const int n = o.nruns[L];
                for (int k = 0; k < n; ++k) push(r[k] & 3u, r[k] >> 2);
            }
        }
        {
            const uint32_t fl = sa.flags[Rt];
            if (fl & SF_EAGER) {
                const int n = (fl >> 8) & 0xff;
                const unsigned long long ops = sa.eops[Rt];
                for (int k = n - 1; k >= 0; --k) push((uint32_t)(ops >> (2 * k)) & 3u, 1);
            } else {
                const uint32_t* r = o.runs + pl.roff[Rt];
                const int n = o.nruns[Rt];
                for (int k = n - 1; k >= 0; --k) push(r[k] & 3u, r[k] >> 2);
            }
        }
        if (len) f(cur, len);
    }
};

__device__ __forceinline__ int ndigits(long long v) {
    int d = 1;
    while (v >= 10) { v /= 10; ++d; }
    return d;
}

__global__ void k_combine_len(Batch b, SideArrays sa, ExecPlan pl, Outputs o, long long* lens) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= b.nseeds) return;
    RunVisitor v{sa, pl, o};
    long long n = 0;
    v.visit(s, [&](uint32_t, long long len) { n += ndigits(len) + 1; });
    lens[s] = n;
}

__global__ void k_combine_total(const long long* offs, const long long* lens, int n, long long* total) {
    if (threadIdx.x == 0 && blockIdx.x == 0) *total = n > 0 ? offs[n - 1] + lens[n - 1] : 0;
}

cudaError_t launch_combine_len(const DevParams&, const Batch& b, const SideArrays& sa, const ExecPlan& pl,
                               const Outputs& o, void* tmp, size_t tmp_bytes, long long* total, cudaStream_t st) {
    const int n = b.nseeds;  // o.cig_len holds 2n entries: offsets [0, n), lengths [n, 2n)
    if (n > 0) {
        k_combine_len<<<(n + 255) / 256, 256, 0, st>>>(b, sa, pl, o, o.cig_len + n);
        size_t bb = tmp_bytes;
        cudaError_t e = cub::DeviceScan::ExclusiveSum(tmp, bb, o.cig_len + n, o.cig_len, n, st);
        if (e != cudaSuccess) return e;
    }
    k_combine_total<<<1, 1, 0, st>>>(o.cig_len, o.cig_len + n, n, total);
    return cudaGetLastError();
}

__global__ void k_combine_write(DevParams P, Batch b, SideArrays sa, ExecPlan pl, Outputs o) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= b.nseeds) return;
    RunVisitor v{sa, pl, o};
    const long long off = o.cig_len[s];
    char* out = o.cigar + off;
    long long n = 0;
    v.visit(s, [&](uint32_t op, long long len) {
        const int d = ndigits(len);
        for (int k = d - 1; k >= 0; --k) {
            out[n + k] = (char)('0' + len % 10);
            len /= 10;
        }
        n += d;
        out[n++] = op == OP_M ? 'M' : (op == OP_I ? 'I' : 'D');
    });
    const int L = 2 * s, Rt = 2 * s + 1;
    const long long tpos = b.seeds[2 * s], qpos = b.seeds[2 * s + 1];
    fastz_alignment a;
    a.left_score = sa.score[L];
    a.right_score = sa.score[Rt];
    a.score = a.left_score + a.right_score;
    const uint32_t fl = sa.flags[L], fr = sa.flags[Rt];
    // eager classification: peak inside the eager window (escalated sides are traced back by the
    // executor even then; the flag reports the classification)
    const bool el = sa.ti[L] <= P.eager_max && sa.qj[L] <= P.eager_max;
    const bool er = sa.ti[Rt] <= P.eager_max && sa.qj[Rt] <= P.eager_max;
    a.flags = (a.score >= P.K ? FASTZ_FLAG_ABOVE_K : 0u) | (el ? FASTZ_FLAG_LEFT_EAGER : 0u) |
              (er ? FASTZ_FLAG_RIGHT_EAGER : 0u) |
              (((fl | fr) & SF_OVERFLOW) ? FASTZ_FLAG_OVERFLOW : 0u) |
              (((fl | fr) & SF_NOTB) ? FASTZ_FLAG_NO_CIGAR : 0u);
    a.t_start = tpos - sa.ti[L];
    a.t_end = tpos + sa.ti[Rt];
    a.q_start = qpos - sa.qj[L];
    a.q_end = qpos + sa.qj[Rt];
    a.cigar_off = off;
    a.cigar_len = (int32_t)n;
    a.reserved = 0;
    reinterpret_cast<fastz_alignment*>(o.recs)[s] = a;
}

cudaError_t launch_combine_write(const DevParams& P, const Batch& b, const SideArrays& sa, const ExecPlan& pl,
                                 const Outputs& o, cudaStream_t st) {
    if (b.nseeds == 0) return cudaSuccess;
    k_combine_write<<<(b.nseeds + 127) / 128, 128, 0, st>>>(P, b, sa, pl, o);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------- launchers
int pick_R() {  // read at fastz_create
    const char* e = getenv("FASTZ_R");
    const int r = e ? atoi(e) : 4;
    return (r == 2 || r == 4) ? r : 4;
}

template <int R>
static int bps_of() {
    int n = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_inspect<R>, WARPS * 32, 0);
    return n > 0 ? n : 1;
}

int inspector_blocks_per_sm(int R) { return R == 2 ? bps_of<2>() : bps_of<4>(); }

#define FZ_DISPATCH(KERNEL, GRID, ...)                                                   \
    do {                                                                                 \
        const bool nm_ = b.TfN || b.QfN; /* N masks present: the N-aware instantiation */ \
        if (R == 2) {                                                                    \
            if (nm_) KERNEL<2, true><<<GRID, WARPS * 32, 0, st>>>(__VA_ARGS__);          \
            else KERNEL<2, false><<<GRID, WARPS * 32, 0, st>>>(__VA_ARGS__);             \
        } else {                                                                         \
            if (nm_) KERNEL<4, true><<<GRID, WARPS * 32, 0, st>>>(__VA_ARGS__);          \
            else KERNEL<4, false><<<GRID, WARPS * 32, 0, st>>>(__VA_ARGS__);             \
        }                                                                                \
    } while (0)

// Inspector escalation of long sides to the block-per-side inspector (FASTZ_ESCALATE_STRIPS, strips; 0 = off).
// Off by default: measured on C1/C2/C3/C5 (profiles/r1_escalation.jsonl) the pipelined block schedule is slower
// than independent warps whenever there are more long sides than warps or none at all -- the inspector cannot
// know lengths in advance, and the warp-per-side queue already hides the long tail.  The executor, which
// knows the lengths, runs bins >= 3 block per side (FASTZ_BLOCK_BIN).
int escalate_strips() {  // read per call: tests and ablations switch it at run time
    const char* e = getenv("FASTZ_ESCALATE_STRIPS");
    int v = e ? atoi(e) : 0;
    return v < 0 ? 0 : v;
}



cudaError_t launch_inspect(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                           const SideArrays& sa, const ExecPlan& pl, int budget, const int* slist, int nlist,
                           cudaStream_t st) {
    if (b.nseeds == 0) return cudaSuccess;
    const bool nm = b.TfN || b.QfN;
    if (R == 2) {
        if (nm) k_inspect_n<2><<<grid, WARPS * 32, 0, st>>>(P, b, ring, rmask, sa, pl, budget, slist, nlist);
        else k_inspect<2><<<grid, WARPS * 32, 0, st>>>(P, b, ring, rmask, sa, pl, budget, slist, nlist);
    } else {
        if (nm) k_inspect_n<4><<<grid, WARPS * 32, 0, st>>>(P, b, ring, rmask, sa, pl, budget, slist, nlist);
        else k_inspect<4><<<grid, WARPS * 32, 0, st>>>(P, b, ring, rmask, sa, pl, budget, slist, nlist);
    }
    return cudaGetLastError();
}

cudaError_t launch_inspect_block(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                                 const SideArrays& sa, const ExecPlan& pl, cudaStream_t st) {
    if (b.nseeds == 0) return cudaSuccess;
    FZ_DISPATCH(k_inspect_block, grid, P, b, ring, rmask, sa, pl);
    return cudaGetLastError();
}

cudaError_t launch_census(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                          long long* cells, int* counter, const int* slist, int nlist, cudaStream_t st) {
    if (b.nseeds == 0) return cudaSuccess;
    FZ_DISPATCH(k_census, grid, P, b, ring, rmask, cells, counter, slist, nlist);
    return cudaGetLastError();
}

cudaError_t launch_execute(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                           const SideArrays& sa, const ExecPlan& pl, int lo, int hi, int nblock, long long base,
                           const Outputs& o, int wide, cudaStream_t st) {
    if (hi <= lo) return cudaSuccess;
    FZ_DISPATCH(k_execute, grid, P, b, ring, rmask, sa, pl, lo, hi, nblock, base, o, wide);
    return cudaGetLastError();
}

cudaError_t launch_traceback(int R, const SideArrays& sa, const ExecPlan& pl, int lo, int hi, int nblock,
                             long long base, const Outputs& o, cudaStream_t st) {
    if (hi <= lo) return cudaSuccess;
    // list positions < nblock hold the long sides (bins >= 3): warp per side with a shared code window
    const int mid = nblock < lo ? lo : (nblock > hi ? hi : nblock);
    if (mid > lo) {
        const int g = (mid - lo + 3) / 4;
        if (R == 2) k_traceback_warp<2><<<g, 128, 0, st>>>(sa, pl, lo, mid, base, o);
        else k_traceback_warp<4><<<g, 128, 0, st>>>(sa, pl, lo, mid, base, o);
    }
    if (hi > mid) {
        const int g = (hi - mid + 127) / 128;
        if (R == 2) k_traceback<2><<<g, 128, 0, st>>>(sa, pl, mid, hi, base, o);
        else k_traceback<4><<<g, 128, 0, st>>>(sa, pl, mid, hi, base, o);
    }
    return cudaGetLastError();
}

}  // namespace fz
