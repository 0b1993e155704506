// pair.cuh -- the packed inspector: two one-sided extensions per warp in the 16-bit halves of every register.
//
// Same strip schedule, hand-off and termination as the SOLO inspector of side.cuh (warp per problem, P:160;
// register rows; strip-boundary ring), but each lane's X / I / W / D registers hold the cells of
// TWO independent sides: side A in the low 16 bits, side B in the high 16 bits.  The halves run their own strips
// (own start column, rows, query, ring, termination, peak) in lockstep steps; a half whose strip has terminated
// keeps computing dead cells (harmless: see DESIGN.md "Packed inspector") until the other half's strip ends, and a
// half whose side has ended takes the next side from the queue at the next strip boundary.
//
// Arithmetic (exact): every value v is stored as v + Z in an unsigned 16-bit half, the
// dead value is NEG_b = max(Y, O+E, E), rows beyond M / columns beyond N carry the threshold BIG_b = NEG_b + 32767.
//   D = max(D_up - E, X_up), I = max(I_left - E, X_left)          VIADDMNMX.U16x2 (per-half add wraps, never below 0)
//   H = X_diag + sub + O + E                                      IMAD (halves >= 0, no carry: the value cap)
//   S = max3(H, D, I)                                             VIMNMX3.U16x2
//   W = max3(S - Y, W_up, W_left)                                 IMAD + VIMNMX3.U16x2 (reading R3's V - Y)
//   live iff S >= W  (== S >= max(W_up, W_left) since Y >= 0)      IADD3 (S - W + 0x8000 per half) + PRMT sign mask
//   X = live ? S - (O+E) : NEG_b                                  IMAD + LOP3
// i.e. 3.5 ALU-pipe + 1.5 FMA-pipe instructions per cell against 6 + 3 for the 32-bit cell of dp.cuh.  A side whose
// peak reaches the value cap (or whose strip outgrows 16-bit step counters) is abandoned here and re-inspected by
// the 32-bit kernel (redo list), so results never depend on the packing.
#pragma once

#include "internal.h"
#include "side.cuh"

namespace fz {


// substitution table of the packed inspector: entry (code, a0, a1) = {sub(a0, code) + OE, sub(a1, code) + OE}
// (values in [0, 2^16)), replicated 16x (conflict-free LDS.64): dp.cuh's SubTab<false> layout, so the fused
// kernel's 32-bit path reads the same table; side A's entry lands in the low half and side B's, multiplied by
// 2^16 in the combining IMAD, in the high half
constexpr int PSUB_CODE = 16 * SUBTAB_ENTRY;     // bytes per query code (4 x 4 row-pair entries)
constexpr int PSUB_TAB = 5 * PSUB_CODE;          // bytes per table (codes 0..4)
constexpr int PSUB_INTS = PSUB_TAB / 4;          // one table: side B's values are shifted by the combining IMAD

struct PairHalf {           // strip-level state of one half (shared memory; lane 0 writes, all lanes read)
    const uint32_t* Apk;
    const uint32_t* Bpk;
    long long Aoff, Boff;
    long long cum_words, bound_words;
    int side, s, M, N;
    int start, Wleft0, lastlive, Emax, Wfar, nfirst;
    int maxsw, bound_maxsw;
    uint32_t flags;
    int active, redo;
    long long t_start, steps;  // diagnostics (FASTZ_PAIR_DEBUG): clock at pop, steps run
};

constexpr int PCP_RING = 64;  // column-code ring of the packed inspector (reads span [t - 31, t + 31])
#ifndef PAIR_TERM
#define PAIR_TERM 32  // steps between strip-termination tests of the packed inspector (8, 16 or 32; measured best 32)
#endif

struct PairWarp {
    int2 co[PCP_RING + BLK];   // column codes of both halves as table byte offsets (+BLK mirrored)
    int4 bin[BLK];            // lane 0's boundary input, packed {X, D, W, -}
    int4 bout[BLK];           // lane 31's bottom-row outputs, packed
    int bi[2][32], bj[2][32]; // per lane and half: peak position (rare slow path)
    int bfirst[2], blast[2];  // per half: first / last live bottom-row column of the current strip (lane 0 writes)
    // per half, current strip: start column, span (N - start), block step at which it began (relative step =
    // tt - t0), termination step (absolute; -1 while running)
    int startv[2], spanv[2], t0v[2], tfin[2];
    PairHalf hs[2];
};

__device__ __forceinline__ unsigned madu(unsigned a, unsigned b, unsigned c) {
    unsigned d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
// a - b + c as one 32-bit IADD3 (exact per half when each half's result stays in [0, 65535])
__device__ __forceinline__ unsigned sub_add(unsigned a, unsigned b, unsigned c) {
    unsigned d;
    asm("{ .reg .u32 t; sub.u32 t, %1, %2; add.u32 %0, t, %3; }" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
// per half: 0xffff if bit 15 of the half is set, else 0 (PRMT sign replication of bytes 1 and 3)
__device__ __forceinline__ unsigned half_sign_mask(unsigned v) {
    unsigned d;
    asm("prmt.b32 %0, %1, 0, 0xBB99;" : "=r"(d) : "r"(v));
    return d;
}
// (a & m) | (n & ~m)
__device__ __forceinline__ unsigned sel_mask(unsigned a, unsigned m, unsigned n) {
    unsigned d;
    asm("lop3.b32 %0, %1, %2, %3, 0xE2;" : "=r"(d) : "r"(a), "r"(m), "r"(n));
    return d;
}
__device__ __forceinline__ unsigned pack2(unsigned lo, unsigned hi) { return (lo & 0xffffu) | (hi << 16); }
__device__ __forceinline__ unsigned half_of(unsigned v, int h) { return h ? (v >> 16) : (v & 0xffffu); }

// boundary row value of half h at column c, stored form: ring entries are int2 {X | D << 16, W}
__device__ __forceinline__ void pair_boundary(const PairHalf& hs, const int2* __restrict__ ring, int rmask, int c,
                                              const PairParams& Q, unsigned& x, unsigned& d, unsigned& w) {
    if (!hs.active) {
        x = d = Q.NEGb;
        w = Q.BIGb;
        return;
    }
    if (c <= hs.Emax) {
        const int2 e = ring[c & rmask];
        x = (unsigned)e.x & 0xffffu;
        d = (unsigned)e.x >> 16;
        w = (unsigned)e.y;
    } else {
        x = d = Q.NEGb;
        w = (unsigned)hs.Wfar;
    }
    if (c > hs.N) w = Q.BIGb;  // columns beyond the query: dead (the 32-bit kernel never computes them)
}

__device__ __forceinline__ int pair_code(const PairHalf& hs, int c) {
    if (!hs.active || c < 1 || c > hs.N) return 4;
    return base_at(hs.Bpk, hs.Boff + c - 1);
}

// Peak update of a packed warp (reading R5: strictly better, or equal in a smaller row; columns only grow): the
// cells of the previous step (p*) and this step (x*) of both halves, in column order.  Returns the new packed
// per-lane peak and flag bits (bit h: half h moved its peak; bit 2 + h: it reached the value cap).
__device__ __noinline__ uint2 pair_peak(PairWarp* ws, unsigned p0, unsigned p1, unsigned p2, unsigned p3, unsigned x0,
                                        unsigned x1, unsigned x2, unsigned x3, unsigned bestP, int tt, unsigned limX) {
    constexpr int R = 4, H = 32 * R;
    const int lane = threadIdx.x & 31;
    const unsigned xs[2][R] = {{p0, p1, p2, p3}, {x0, x1, x2, x3}};
    unsigned flg = 0;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        const int c = ws->startv[h] - ws->t0v[h] + tt - lane;
        const int r0 = ws->hs[h].s * H + lane * R;
        unsigned best = half_of(bestP, h);
        int bi = ws->bi[h][lane], bj = ws->bj[h][lane];
        bool any = false;
#pragma unroll
        for (int q = 0; q < 2; ++q) {
#pragma unroll
            for (int k = 0; k < R; ++k) {
                const unsigned x = half_of(xs[q][k], h);
                const int r = r0 + k;
                const bool better = x > best || (x == best && r < bi);
                best = better ? x : best;
                bi = better ? r : bi;
                bj = better ? c - 1 + q : bj;
                any |= better;
            }
        }
        if (any) {
            const unsigned hm = h ? 0xffff0000u : 0x0000ffffu;
            bestP = (bestP & ~hm) | (best * 0x10001u & hm);
            ws->bi[h][lane] = bi;
            ws->bj[h][lane] = bj;
            flg |= (best >= limX ? 5u : 1u) << h;
        }
    }
    return make_uint2(bestP, flg);
}

template <int R>
__device__ __forceinline__ bool run_pairs(const DevParams& P, const PairParams& Q, const Batch& b, int2* ring_base,
                                          int rmask, const SideArrays& sa, const ExecPlan& pl, PairWarp* ws,
                                          unsigned subtab, const int* __restrict__ slist, int nsides, int* queue,
                                          long long* dbg = nullptr, int* own = nullptr) {
    static_assert(R == 4, "the packed inspector runs 4 rows per lane");
    constexpr int H = StripGeom<R>::H;
    constexpr int SPW = StripGeom<R>::SPW;
    constexpr int BK = BLK;
    const int lane = threadIdx.x & 31;
    const int src = (lane + 31) & 31;
    const bool is31 = lane == 31, is0 = lane == 0;
    const unsigned one = (unsigned)P.one;
    const unsigned NEG2 = Q.NEGb * 0x10001u, K8 = 0x80008000u;
    const unsigned NEG1P = (Q.NEGb + 1u) * 0x10001u;
    const unsigned sb_in = (unsigned)__cvta_generic_to_shared(&ws->bin[0]);
    const unsigned sb_out = (unsigned)__cvta_generic_to_shared(&ws->bout[0]);
    const unsigned co_base = (unsigned)__cvta_generic_to_shared(&ws->co[0]);
    auto ringh = [&](int h) { return ring_base + (h ? rmask + 1 : 0); };
    auto hmask = [](int h) { return h ? 0xffff0000u : 0x0000ffffu; };
    auto merge = [](unsigned v, unsigned nv, unsigned hm) { return (v & ~hm) | (nv & hm); };

    // take the next side for half h (all lanes; lane 0 owns the queue and the shared state)
    // own (mixed kernel): a pending redo side this warp has claimed (-1: none); while it owns one the warp takes no
    // new packed sides, so it returns to the 32-bit inspector as soon as both halves are idle
    auto pop = [&](int h) {
        int side = 0;
        if (lane == 0) {
            if (own) {
                volatile int* ctr = pl.counters;
                if (*own < 0) {
                    int c = ctr[34];
                    while (c < ctr[30]) {
                        const int o = atomicCAS(&pl.counters[34], c, c + 1);
                        if (o == c) {
                            *own = c;
                            break;
                        }
                        c = o;
                    }
                }
            }
            side = (own && *own >= 0) ? nsides : atomicAdd(queue, 1);
        }
        __syncwarp();
        side = __shfl_sync(FULL, side, 0);
        PairHalf& hs = ws->hs[h];
        __syncwarp();
        if (lane == 0) {
            if (side >= nsides) {
                hs.active = 0;
                hs.N = -1;
                hs.M = -1;
                hs.s = 0;
            } else {
                if (slist) side = slist[side];
                SideIO io;
                setup_side<false>(b, side, io);
                hs.Apk = io.Apk;
                hs.Aoff = io.Aoff;
                hs.M = io.M;
                hs.Bpk = io.Bpk;
                hs.Boff = io.Boff;
                hs.N = io.N;
                hs.side = side;
                hs.s = 0;
                hs.start = 0;
                hs.Wleft0 = (int)((unsigned)Q.WoutT + Q.Z);
                hs.lastlive = -1;
                hs.Emax = -1;
                hs.Wfar = (int)Q.NEGb;
                hs.nfirst = INT_MAX;
                hs.cum_words = hs.bound_words = 0;
                hs.maxsw = hs.bound_maxsw = 0;
                hs.flags = 0;
                hs.active = 1;
                hs.redo = 0;
                hs.t_start = clock64();
                hs.steps = 0;
            }
        }
        ws->bi[h][lane] = INT_MAX;
        ws->bj[h][lane] = INT_MAX;
        __syncwarp();
    };

    // registers: both halves' cells; per half: strip start column, span (N - start), the block step at which the
    // strip began (relative step = tt - t0), termination step (absolute, -1 while running)
    unsigned X[R], I[R], W[R], Xp[R];
    unsigned tb[2][R / 2];
    unsigned xdiag, cacc, lastlive_t, bestP = NEG1P;
    uint4 bq;
    int* const startv = ws->startv;
    int* const spanv = ws->spanv;
    int* const t0v = ws->t0v;
    int* const tfin = ws->tfin;
    unsigned flg = 0;  // bit h: lane moved half h's peak in this strip; bit 2 + h: half h reached the value cap
#pragma unroll
    for (int k = 0; k < R; ++k) X[k] = I[k] = W[k] = Xp[k] = NEG2;
    xdiag = cacc = NEG2;
    lastlive_t = 0;
    bq = make_uint4(NEG2, NEG2, NEG2, 0);

    // new strip of half h from block step t (its PairHalf is current): registers of half h only
    auto setup_half = [&](int h, int t) {
        const PairHalf& hs = ws->hs[h];
        const unsigned hm = hmask(h);
        const int top = hs.s * H;
        const int r0 = top + lane * R;
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const int r = r0 + k;
            int a = 0;
            if (hs.active && r >= 1 && r <= hs.M) a = base_at(hs.Apk, hs.Aoff + r - 1);
            const unsigned base = subtab + (unsigned)((lane & 15) * 8);
            if (k % 2 == 0) tb[h][k / 2] = base + (unsigned)(a * 4 * SUBTAB_ENTRY);
            else tb[h][k / 2] += (unsigned)(a * SUBTAB_ENTRY);
            const unsigned wv = (hs.active && r <= hs.M) ? (unsigned)hs.Wleft0 : Q.BIGb;
            W[k] = merge(W[k], wv * 0x10001u, hm);
            X[k] = merge(X[k], NEG2, hm);
            I[k] = merge(I[k], NEG2, hm);
            Xp[k] = merge(Xp[k], NEG2, hm);
        }
        // origin: H(0,0) = -OE + 0 + OE = 0
        const unsigned xo = (hs.active && top == 0 && lane == 0) ? Q.Z - (unsigned)P.OE : Q.NEGb;
        xdiag = merge(xdiag, xo * 0x10001u, hm);
        bq.x = merge(bq.x, NEG2, hm);
        bq.y = merge(bq.y, NEG2, hm);
        bq.z = merge(bq.z, NEG2, hm);
        cacc = merge(cacc, NEG2, hm);
        lastlive_t &= ~hm;
        flg &= ~(1u << h);
        __syncwarp();
        if (lane == 0) {
            startv[h] = hs.active ? hs.start : 0;
            spanv[h] = hs.active ? hs.N - hs.start : -1;
            t0v[h] = t;
            tfin[h] = hs.active ? -1 : t - 1;
            ws->bfirst[h] = INT_MAX;
            ws->blast[h] = -1;
        }
        __syncwarp();
    };

    // park lane 31's outputs of steps [st0, st0 + 31] into the halves' rings (half h up to step stmax_h)
    auto park = [&](int st0, int stmax0, int stmax1) {
        const int st = st0 + lane;
        const int4 v = ws->bout[st & (BK - 1)];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int rc31 = st - t0v[h] - 31;
            const bool ok = st <= (h ? stmax1 : stmax0) && rc31 >= 0 && rc31 <= spanv[h];
            const unsigned xv = half_of((unsigned)v.x, h);
            if (ok) {
                const unsigned dv = half_of((unsigned)v.y, h), wv = half_of((unsigned)v.z, h);
                ringh(h)[(startv[h] + rc31) & rmask] = make_int2((int)(xv | (dv << 16)), (int)wv);
            }
            const unsigned bal = __ballot_sync(FULL, ok && xv != Q.NEGb);
            if (bal && lane == 0) {
                const int c0 = startv[h] + st0 - t0v[h] - 31;
                if (ws->bfirst[h] == INT_MAX) ws->bfirst[h] = c0 + __ffs(bal) - 1;
                ws->blast[h] = c0 + 31 - __clz(bal);
            }
        }
    };

    // strip finish of half h (its strip terminated at step tfin[h]); returns after the next strip / side is set
    // up in the shared state (the caller then runs setup_half)
    auto finish = [&](int h) {
        PairHalf& hs = ws->hs[h];
        const bool anyupd = __any_sync(FULL, (flg >> h) & 1u);
        int2* __restrict__ rg = ringh(h);
        const int start = startv[h], tf = tfin[h] - t0v[h];
        const int e = start + tf - 31;  // lane 31's last column
        int2* const hist = Q.hist ? Q.hist + ((size_t)(blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + h) *
                                                 PAIR_HIST
                                  : nullptr;
        if (lane == 0) {
            hs.steps += tf + 1;
            if (hist && hs.s < PAIR_HIST) hist[hs.s] = make_int2(start, tf);
        }
        bool over = hs.redo != 0;
        int Emax = hs.Emax, Wfar = hs.Wfar;
        uint32_t flags = hs.flags;
        long long cum_words = hs.cum_words, bound_words = hs.bound_words;
        int maxsw = hs.maxsw, bound_maxsw = hs.bound_maxsw;
        if (!over) {
            const int sw = (tf / SPW + 1) * 32;
            const int maxsw_prev = maxsw;
            cum_words += sw;
            maxsw = sw > maxsw ? sw : maxsw;
            if (anyupd) {  // executor storage bound (side.cuh)
                int mbj = ws->bj[h][lane] == INT_MAX ? 0 : ws->bj[h][lane];
#pragma unroll
                for (int off = 16; off; off >>= 1) mbj = imax(mbj, __shfl_xor_sync(FULL, mbj, off));
                const int sp = mbj - start > 0 ? mbj - start : 0;
                const int tt2 = tf < sp + 31 ? tf : sp + 31;
                const int tw = (tt2 / SPW + 1) * 32;
                const int wj = ((mbj + 31) / SPW + 1) * 32;
                const long long above = cum_words - sw;
                const long long cap = (long long)hs.s * wj;
                bound_words = (above < cap ? above : cap) + tw;
                bound_maxsw = imax(maxsw_prev < wj ? maxsw_prev : wj, tw);
            }
            if (e - start + 4 > rmask) {  // strip wider than the ring
                flags |= SF_RING;
                over = true;
            }
            if (hs.s + 1 >= Q.esc_strips) {  // a long side: redo it in 32 bits
                if (lane == 0) hs.redo = 1;
                over = true;
            }
            if (!over) {
                const int Wtail = rg[e & rmask].y;  // W of the bottom row at column e (parked)
                __syncwarp();
                for (int c = e + 1 + lane; c <= Emax; c += 32) {
                    const int2 v = rg[c & rmask];
                    rg[c & rmask] = make_int2((int)NEG2, imax(v.y, Wtail));
                }
                if (e >= Emax) {
                    Emax = e;
                    Wfar = Wtail;
                } else {
                    Wfar = imax(Wfar, Wtail);
                }
                if (hs.s * H + H > hs.M || ws->blast[h] < 0) over = true;  // matrix bottom / no live cell (R6)
                if (!over && Emax + 4 - ws->bfirst[h] > rmask) {
                    flags |= SF_RING;
                    over = true;
                }
            }
        }
        __syncwarp();
        if (!over) {
            const int nf = ws->bfirst[h];
            const int Wl = nf > start ? rg[(nf - 1) & rmask].y : hs.Wleft0;
            __syncwarp();
            if (lane == 0) {
                hs.Emax = Emax;
                hs.Wfar = Wfar;
                hs.flags = flags;
                hs.cum_words = cum_words;
                hs.bound_words = bound_words;
                hs.maxsw = maxsw;
                hs.bound_maxsw = bound_maxsw;
                hs.lastlive = ws->blast[h];
                hs.nfirst = nf;
                hs.start = nf;
                hs.Wleft0 = Wl;
                hs.s = hs.s + 1;
            }
            __syncwarp();
            return;
        }
        // side done: peak over the warp (ties: min i, then min j)
        int best = (int)half_of(bestP, h), bi = ws->bi[h][lane], bj = ws->bj[h][lane];
#pragma unroll
        for (int off = 16; off; off >>= 1) {
            const int ob = __shfl_xor_sync(FULL, best, off);
            const int oi = __shfl_xor_sync(FULL, bi, off);
            const int oj = __shfl_xor_sync(FULL, bj, off);
            if (ob > best || (ob == best && (oi < bi || (oi == bi && oj < bj)))) {
                best = ob;
                bi = oi;
                bj = oj;
            }
        }
        if (lane == 0) {
            const int side = hs.side;
            if (dbg) {
                dbg[4 * side] = clock64() - hs.t_start;
                dbg[4 * side + 1] = hs.s + 1;
                dbg[4 * side + 2] = hs.steps;
                dbg[4 * side + 3] = hs.redo ? 1 : 0;
            }
            if (hs.redo) {
                pl.redo[atomicAdd(&pl.counters[30], 1)] = side;
            } else {
                const bool notrim = P.options & OPT_NO_TRIM;
                const int nstr = hs.s + 1;
                // Exact executor storage ("allocate ... according to the exact size needed"): the executor's
                // strip k (k <= i*/H) starts at the same column as the inspector's and runs at most
                // min(inspector steps, j* - start_k + 31) steps, so its words are bounded by that width exactly.
                const int speak = bi / H;
                if (hist && !notrim && speak <= hs.s && speak < PAIR_HIST) {
                    long long words = 0;
                    int mx = 0;
                    for (int k = 0; k <= speak; ++k) {
                        const int2 hk = hist[k];
                        const int sp = bj - hk.x > 0 ? bj - hk.x : 0;
                        const int wk = ((hk.y < sp + 31 ? hk.y : sp + 31) / SPW + 1) * 32;
                        words += wk;
                        mx = wk > mx ? wk : mx;
                    }
                    bound_words = words;
                    bound_maxsw = mx;
                }
                sa.score[side] = best - (int)Q.Z + P.OE;
                sa.ti[side] = bi;
                sa.qj[side] = bj;
                sa.flags[side] = flags | SF_PAIR;
                sa.eops[side] = 0ull;
                sa.bound[side] = notrim ? cum_words : bound_words;
                sa.maxsw[side] = notrim ? maxsw : bound_maxsw;
                sa.nstrip[side] = notrim ? nstr : -1;
            }
        }
        bestP = merge(bestP, NEG1P, hmask(h));
        flg &= ~(4u << h);
        pop(h);
    };

    // boundary + column codes of half h for relative columns rc (this lane's entry), stored form
    auto stage_half = [&](int h, int rc, unsigned& x, unsigned& d, unsigned& w, int& co) {
        const PairHalf& hs = ws->hs[h];
        pair_boundary(hs, ringh(h), rmask, startv[h] + rc, Q, x, d, w);
        co = pair_code(hs, startv[h] + rc) * PSUB_CODE;
    };

    // the column-code ring is read ahead of a strip's first column during ramp-up (dead cells): valid offsets
    for (int i = lane; i < PCP_RING + BLK; i += 32) ws->co[i] = make_int2(4 * PSUB_CODE, 4 * PSUB_CODE);
    pop(0);
    pop(1);
    setup_half(0, 0);
    setup_half(1, 0);

    // one wavefront step: lane computes relative column tt - t0_h - lane of each half
    auto step = [&](const int tt, const int j, const unsigned coa, const unsigned sgo, const unsigned sgi,
                    const unsigned ttbase) {
        int xu_ = (int)__shfl_sync(FULL, bq.x, src);
        int du_ = (int)__shfl_sync(FULL, bq.y, src);
        int wu_ = (int)__shfl_sync(FULL, bq.z, src);
        // lane 0 replaces what lane 31 sent with the boundary row of both halves
        ld_shared3_if(is0, sgi + 16u * (unsigned)j, xu_, du_, wu_);
        unsigned xu = (unsigned)xu_, du = (unsigned)du_, wu = (unsigned)wu_;
        int cA, cB;
        ld_shared2((int)coa, cA, cB);
        unsigned w[R];
#pragma unroll
        for (int p = 0; p < R / 2; ++p) {
            int l0, l1, h0, h1;
            ld_shared2(fma_add(cA, (int)one, (int)tb[0][p]), l0, l1);
            ld_shared2(fma_add(cB, (int)one, (int)tb[1][p]), h0, h1);
            w[2 * p] = madu((unsigned)h0, 0x10000u, (unsigned)l0);  // {sub_A, sub_B} halves (no carry: < 2^16)
            w[2 * p + 1] = madu((unsigned)h1, 0x10000u, (unsigned)l1);
        }
        unsigned xd = xdiag;
        xdiag = xu;
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const unsigned hv = madu(w[k], one, xd);              // X_diag + sub + O + E
            const unsigned d = __viaddmax_u16x2(du, Q.mE2, xu);   // max(D_up - E, X_up)
            const unsigned iv = __viaddmax_u16x2(I[k], Q.mE2, X[k]);
            const unsigned sr = __vimax3_u16x2(hv, d, iv);
            const unsigned sy = madu(sr, one, Q.mY2);              // S - Y
            const unsigned wn = __vimax3_u16x2(sy, wu, W[k]);      // V - Y (reading R3)
            const unsigned lm = half_sign_mask(sub_add(sr, wn, K8));  // live iff S >= W
            const unsigned xn = sel_mask(madu(sr, one, Q.mOE2), lm, NEG2);
            xd = X[k];
            X[k] = xn;
            I[k] = iv;
            W[k] = wn;
            xu = xn;
            du = d;
            wu = wn;
        }
        bq.x = xu;
        bq.y = du;
        bq.z = wu;
        cacc = __vimax3_u16x2(cacc, X[0], X[1]);
        cacc = __vimax3_u16x2(cacc, X[2], X[3]);
        if ((j & 1) == 0) {
#pragma unroll
            for (int k = 0; k < R; ++k) Xp[k] = X[k];
        } else if (__any_sync(FULL, (sub_add(cacc, bestP, K8) & K8) != 0u)) {
            // peak (reading R5), rare: an out-of-line scan of both steps' cells of both halves, so the fast path's
            // registers are not pinned around the branch
            const uint2 r = pair_peak(ws, Xp[0], Xp[1], Xp[2], Xp[3], X[0], X[1], X[2], X[3], bestP, tt, Q.limX);
            bestP = r.x;
            flg |= r.y;
        }
        // lane 31 parks its bottom row
        st_shared4_if(is31, sgo + 16u * (unsigned)j, make_int4((int)bq.x, (int)bq.y, (int)bq.z, 0));
        if (j == 3) {
            // liveness per 4-step group and half: live anywhere in the group -> (relative group end step) + 1
            const unsigned lm = half_sign_mask(sub_add(cacc, NEG1P, K8));
            lastlive_t = sel_mask(madu((unsigned)tt, 0x10001u, ttbase), lm, lastlive_t);
            cacc = NEG2;
        }
    };
    // strip termination of the halves at a test step (relative step = 7 mod 8 and >= 31: the SOLO test points)
    auto term = [&](const int tt) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int rel = tt - t0v[h];
            if (tfin[h] < 0 && rel >= 31) {
                int tf = -1;
                if (rel >= spanv[h] + 31) {  // lane 31 reached column N (the 32-bit kernel's tlast)
                    tf = t0v[h] + spanv[h] + 31;
                } else {
                    const unsigned bal = __ballot_sync(FULL, (int)half_of(lastlive_t, h) < rel - 30 + lane);
                    if (bal == FULL && startv[h] + rel - 31 > ws->hs[h].lastlive) tf = tt;
                }
                __syncwarp();
                if (lane == 0 && tf >= 0) tfin[h] = tf;
                __syncwarp();
            }
        }
    };

    for (int t = 0;; t += BK) {
        if (t > 0) {
            __syncwarp();
            park(t - BK, tfin[0] >= 0 ? tfin[0] : t - 1, tfin[1] >= 0 ? tfin[1] : t - 1);
            __syncwarp();
            const unsigned capped = __ballot_sync(FULL, (flg >> 2) & 1u) ? 1u : 0u;
            const unsigned capped1 = __ballot_sync(FULL, (flg >> 3) & 1u) ? 2u : 0u;
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                if (!ws->hs[h].active) continue;
                // value cap reached, or a strip beyond the 16-bit step counters: abandon (redone in 32 bits)
                if (((capped | capped1) >> h) & 1u || (tfin[h] < 0 && t - t0v[h] > 65000)) {
                    __syncwarp();
                    if (lane == 0) {
                        ws->hs[h].redo = 1;
                        if (tfin[h] < 0) tfin[h] = t - 1;
                    }
                    __syncwarp();
                }
                if (tfin[h] >= 0) {
                    finish(h);
                    setup_half(h, t);
                }
            }
            __syncwarp();
        }
        if (!(ws->hs[0].active | ws->hs[1].active)) return !(own && *own >= 0);  // true: the packed queue is empty
        // staging: boundary entries and column codes of steps [t, t + BK)
        {
            unsigned x0, d0, w0, x1, d1, w1;
            int c0, c1;
            stage_half(0, t - t0v[0] + lane, x0, d0, w0, c0);
            stage_half(1, t - t0v[1] + lane, x1, d1, w1, c1);
            ws->bin[lane] = make_int4((int)pack2(x0, x1), (int)pack2(d0, d1), (int)pack2(w0, w1), 0);
            const int idx = (t + lane) & (PCP_RING - 1);
            ws->co[idx] = make_int2(c0, c1);
            if (idx < BLK) ws->co[idx + PCP_RING] = make_int2(c0, c1);
        }
        __syncwarp();
        const unsigned cob = co_base + 8u * (unsigned)((t - lane) & (PCP_RING - 1));
        // relative group-end step + 1 of both halves: tt * 0x10001 + ttbase
        const unsigned ttbase = 0x10001u - ((unsigned)t0v[0] | ((unsigned)t0v[1] << 16));
#pragma unroll 1
        for (int q = 0; q < BK; q += STEADY_UNROLL) {
            const unsigned sgo = sb_out + 16u * (unsigned)q, sgi = sb_in + 16u * (unsigned)q;
            const unsigned coq = cob + 8u * (unsigned)q;
#pragma unroll
            for (int u = 0; u < STEADY_UNROLL; ++u)
                step(t + q + u, u & 3, coq + 8u * (unsigned)u, sgo + 16u * (unsigned)(u & ~3),
                     sgi + 16u * (unsigned)(u & ~3), ttbase);
            if ((q & (PAIR_TERM - 8)) == (PAIR_TERM - 8)) {
                // strip termination every PAIR_TERM steps (relative step PAIR_TERM - 1 mod PAIR_TERM; the SOLO kernel
                // tests every 8): a later test only computes and parks more cells that are dead either way (past
                // the termination column every cell of the strip is dead; their parked W is the exact V - Y), so
                // results are unchanged while the two halves' ballots, shared loads and syncs run 4x less often
                term(t + q + STEADY_UNROLL - 1);
                if (tfin[0] >= 0 && tfin[1] >= 0) break;  // both strips done: finish them at once
            }
        }
    }
    return true;
}

}  // namespace fz
