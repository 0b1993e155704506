// side.cuh -- one warp runs one one-sided extension, strip by strip (see dp.cuh for the layout).
//
// MODE_INSPECT: score-only pass that finds the peak ("lightweight inspector"), records the 17x17 corner
//               codes during the first steps of strip 0 for eager traceback, and bounds the
//               executor's traceback storage (the executor's allocation is sized by the inspector).
// MODE_EXEC:    the trimmed executor: the same DP restricted to [0,i*]x[0,j*] (exact, because the cone
//               rule of reading R3 only looks inside the rectangle), writing 4-bit codes to HBM in a
//               step-major layout: word (t / SPW) * 32 + lane of the strip holds lane's R rows for SPW steps,
//               so each warp store is one coalesced 128-byte line (P:180's consolidation, done in registers).
// MODE_CENSUS:  counts explored cells (origin + cells with a live diagonal/up/left neighbour), the GCUPS
//               numerator; not on the timed path.
//
// Per-step data movement (the paper's register exchange, re-designed for sm_100a):
//  * lane l receives the bottom row (X, D, W) of lane l-1 with a ROTATING shuffle (src = l-1 mod 32): lane 0
//    receives from lane 31, which -- after parking its own bottom row in shared staging -- holds the previous
//    strip's boundary value for lane 0's next column.  No per-step global memory access, no lane-0 selects.
//  * every 16 steps the warp moves 16 boundary values global ring -> shared staging (prefetched one block
//    ahead) and 16 parked bottom-row values shared -> global ring, both coalesced.
//  * termination: each lane keeps the last step at which one of its R cells was live; the strip is done at
//    column x (lane 31's) iff no lane has had a live cell since it processed x and the boundary row has no
//    live cell at or after x -- the unrolled form of the per-lane "done" chain (lane l is done at x iff its
//    cells are dead at x and lane l-1 is done at x).  Tested every 4 steps.
#pragma once
#include <type_traits>

#include "dp.cuh"

namespace fz {

enum { MODE_INSPECT = 0, MODE_EXEC = 1, MODE_CENSUS = 2 };

struct WarpSmem {
    int2 cp[CP_RING + 16];  // column profiles, ring over relative columns (+16 mirrored)
    int bin[3][32];         // boundary row staging (X, D, W; lane 0's input, served through lane 31)
    int bout[3][32];        // lane 31's bottom-row outputs (X, D, W) awaiting the global ring
};

struct SideIO {
    const uint32_t* __restrict__ Apk;  // target side (rows), packed; A_k at position Aoff + k - 1
    int64_t Aoff;
    int M;                              // rows 0..M
    const uint32_t* __restrict__ Bpk;  // query side (columns)
    int64_t Boff;
    int Bmax;                           // real query length (bases beyond are never read)
    int N;                              // columns 0..N (N <= Bmax; the executor trims to j*)
    int4* __restrict__ ring;            // per-warp boundary ring, rmask + 1 entries {X, D, W, -}
    int rmask;
    WarpSmem* ws;                       // shared staging of this warp
    const int2* cptab;                  // shared: 5 profiles (query base 0..3, zero)
    uint8_t* ecodes;                    // shared: EAGER_W^2 eager codes (inspector)
    int eager_max;
    uint32_t* __restrict__ codes;       // executor: the side's code words
    int2* __restrict__ stab;            // executor: per strip {start column, word offset}
};

struct SideOut {
    int best, bi, bj;        // peak in X space (score = best + O + E), ties: min i, min j
    uint32_t flags;
    long long bound_words;   // inspector: executor words up to the peak strip
    long long cells;         // census: explored cells (warp total)
    long long words;         // executor: words written
};

template <int R>
struct StripGeom {
    static constexpr int H = 32 * R;
    static constexpr int SPW = 8 / R;  // steps per 32-bit code word
};

__device__ __forceinline__ int query_code(const SideIO& io, int c) {
    return (c >= 1 && c <= io.N) ? base_at(io.Bpk, io.Boff + c - 1) : 4;
}

__device__ __forceinline__ void cp_store(const SideIO& io, int rc, int code) {
    const int2 v = io.cptab[code];
    const int idx = rc & (CP_RING - 1);
    io.ws->cp[idx] = v;
    if (idx < 16) io.ws->cp[idx + CP_RING] = v;
}

__device__ __forceinline__ int4 boundary(const int4* __restrict__ ring, int rmask, int c, int Emax, int Wfar) {
    return c <= Emax ? ring[c & rmask] : make_int4(NEG, NEG, Wfar, 0);
}

template <int R, int MODE, bool EAGER, bool FOLD>
__device__ __forceinline__ void run_side(const DevParams& P, const SideIO& io, SideOut& out) {
    constexpr int H = StripGeom<R>::H;
    constexpr int SPW = StripGeom<R>::SPW;
    const int lane = threadIdx.x & 31;
    const int src = (lane + 31) & 31;
    const int M = io.M, N = io.N;
    const int E = P.E, OE = P.OE, OEmY = P.OE - P.Y, mE = -P.E, mOE = -P.OE;
    const int one = P.one, zero = P.zero;
    const int rmask = io.rmask;
    int4* __restrict__ ring = io.ring;
    WarpSmem* __restrict__ ws = io.ws;
    const bool is31 = lane == 31;
    const unsigned sb_in = (unsigned)__cvta_generic_to_shared(&ws->bin[0][0]);
    const unsigned sb_out = (unsigned)__cvta_generic_to_shared(&ws->bout[0][0]);

    // W left of column 0 is V(i,-1) - Y = -inf; any value <= -Y gives the same thresholds (only the origin has
    // no finite neighbour, and it is live for any threshold <= 0).  -(Y+1) keeps the cells that lanes compute
    // before the strip's first column (ramp-up, left of column 0) dead, so ramp-up runs unchecked.
    const int Wout = -P.Y - 1;
    int start = 0, Wleft0 = Wout, lastlive = -1, Emax = -1, Wfar = NEG;
    int best = NEG + 1, bi = INT_MAX, bj = INT_MAX;
    long long cum_words = 0, bound_words = 0, cells = 0;
    uint32_t flags = 0;
    bool upd = false;

    int s = 0;
    for (int top = 0; top <= M; top += H, ++s) {
        // ------------------------------------------------------------------ strip set-up
        int sel[R], X[R], I[R], W[R];
        const int r0 = top + lane * R;
        int nvalid = M - r0 + 1;
        nvalid = nvalid < 0 ? 0 : (nvalid > R ? R : nvalid);
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const int r = r0 + k;
            int a = 0;
            if (r >= 1 && r <= M) a = base_at(io.Apk, io.Aoff + r - 1);
            sel[k] = row_selector(a);
            X[k] = NEG;
            I[k] = NEG;
            W[k] = (r <= M) ? Wleft0 : BIG;
        }
        int xdiag = (top == 0 && lane == 0) ? -OE : NEG;  // origin: H(0,0) = -OE + 0 + OE = 0
        int xb = NEG, db = NEG, wb = NEG;
        const int span = N - start;
        const int tlast = span + 31;
        const long long wbase = cum_words;  // executor: this strip's first word (relative to the side)
        if constexpr (MODE == MODE_EXEC) {
            if (lane == 0) io.stab[s] = make_int2(start, (int)wbase);
        }
        // staging: boundary for relative columns [0, 32), column profiles [0, 32); prefetch the next 16
        {
            const int4 v = boundary(ring, rmask, start + lane, Emax, Wfar);
            ws->bin[0][lane] = v.x;
            ws->bin[1][lane] = v.y;
            ws->bin[2][lane] = v.z;
        }
        cp_store(io, lane, query_code(io, start + lane));
        int4 bpre = make_int4(NEG, NEG, Wfar, 0);
        int qpre = 4;
        if (lane < 16) {
            bpre = boundary(ring, rmask, start + 32 + lane, Emax, Wfar);
            qpre = query_code(io, start + 32 + lane);
        }
        __syncwarp();
        if (lane == 31) {
            xb = ws->bin[0][0];
            db = ws->bin[1][0];
            wb = ws->bin[2][0];
        }
        uint32_t cw = 0;
        int lastlive_t = -1;   // last step at which this lane had a live cell (termination, see header)
        int tfinal = 0;

        // one wavefront step: lane computes column start + tt - lane.  Returns true when the strip is done.
        auto step = [&](auto chk, auto eag, const int tt, const int u, const int j, const int cbase) -> bool {
            constexpr bool CHK = decltype(chk)::value;
            constexpr bool EG = decltype(eag)::value;
            const int rc = tt - lane;
            const bool valid = CHK ? (unsigned)rc <= (unsigned)span : true;
            int xu = __shfl_sync(FULL, xb, src);
            int du = __shfl_sync(FULL, db, src);
            int wu = __shfl_sync(FULL, wb, src);
            int cmv = NEG;
            if (valid) {
                const int2 cp = ws->cp[cbase + u];
                int xd = xdiag;
                xdiag = xu;
                int cm = NEG;
#pragma unroll
                for (int k = 0; k < R; ++k) {
                    const int h = FOLD ? fma_add(prmt(cp.x, cp.y, sel[k]), one, xd)
                                       : xd + prmt(cp.x, cp.y, sel[k]) + OE;
                    const int d = __viaddmax_s32(du, mE, xu);
                    const int iv = __viaddmax_s32(I[k], mE, X[k]);
                    const int sr = __vimax3_s32(h, d, iv);
                    const int thr = imax(wu, W[k]);
                    const int xn = kill_fma(sr, thr, mOE, one, zero);
                    const int wn = __viaddmax_s32(xn, OEmY, thr);
                    if constexpr (MODE == MODE_EXEC) {
                        const uint32_t code = cell_code(h, d, iv, du, xu, I[k], X[k], E);
                        cw |= code << ((((j % SPW) * R) + k) * 4);
                    }
                    if constexpr (EG) {
                        const int r = r0 + k, c = start + rc;
                        if (r <= io.eager_max && c <= io.eager_max)
                            io.ecodes[r * EAGER_W + c] = (uint8_t)cell_code(h, d, iv, du, xu, I[k], X[k], E);
                    }
                    if constexpr (MODE == MODE_CENSUS) {
                        cells += (k < nvalid) && ((xd != NEG) | (xu != NEG) | (X[k] != NEG));
                    }
                    xd = X[k];
                    X[k] = xn;
                    I[k] = iv;
                    W[k] = wn;
                    xu = xn;
                    du = d;
                    wu = wn;
                    cm = k == 0 ? xn : imax(cm, xn);
                }
                xb = xu;
                db = du;
                wb = wu;
                // live -> tt, dead (cm == NEG) -> -1: one VIADDMNMX (min) + one max
                lastlive_t = imax(lastlive_t, __viaddmin_s32(cm, -NEG - 1, tt));
                cmv = cm;
            }
            if constexpr (MODE == MODE_INSPECT) {
                // peak (reading R5): rare, warp-uniform slow path; ties -> smaller row (columns only grow)
                if (__any_sync(FULL, cmv >= best)) {
                    const int c = start + rc;
#pragma unroll
                    for (int k = 0; k < R; ++k) {
                        const int r = r0 + k;
                        const bool better = valid && (X[k] > best || (X[k] == best && r < bi));
                        best = better ? X[k] : best;
                        bi = better ? r : bi;
                        bj = better ? c : bj;
                        upd |= better;
                    }
                }
            }
            {
                const unsigned o = (unsigned)(tt & 31) * 4u, n = (unsigned)((tt + 1) & 31) * 4u;
                st_shared_if(is31, sb_out + o, xb);
                st_shared_if(is31, sb_out + 128u + o, db);
                st_shared_if(is31, sb_out + 256u + o, wb);
                ld_shared_if(is31, sb_in + n, xb);
                ld_shared_if(is31, sb_in + 128u + n, db);
                ld_shared_if(is31, sb_in + 256u + n, wb);
            }
            if constexpr (MODE == MODE_EXEC) {
                if ((j % SPW) == SPW - 1) {  // j == tt mod 4 and SPW divides 4
                    io.codes[wbase + (long long)(tt / SPW) * 32 + lane] = cw;
                    cw = 0;
                }
            }
            if (j == 3 && tt >= 31) {
                // done at lane 31's column x = start + tt - 31 iff every lane has been dead since it processed
                // x (step tt - 31 + lane) and the boundary row has no live cell at or after x
                const unsigned bal = __ballot_sync(FULL, lastlive_t < tt - 31 + lane);
                if (bal == FULL && start + tt - 31 > lastlive) {
                    tfinal = tt;
                    return true;
                }
            }
            if (CHK && tt == tlast) {
                tfinal = tt;
                return true;
            }
            return false;
        };

        int t = 0;
        for (;;) {
            if (t > 0) {
                __syncwarp();  // lane 31's parked rows of the previous block -> visible to lanes 0..15
                // staging refills for relative columns [t+16, t+32), prefetch [t+32, t+48); park -> ring
                if (lane < 16) {
                    const int rcn = t + 16 + lane;
                    ws->bin[0][rcn & 31] = bpre.x;
                    ws->bin[1][rcn & 31] = bpre.y;
                    ws->bin[2][rcn & 31] = bpre.z;
                    cp_store(io, rcn, qpre);
                    bpre = boundary(ring, rmask, start + rcn + 16, Emax, Wfar);
                    qpre = query_code(io, start + rcn + 16);
                    const int st = t - 16 + lane, rc31 = st - 31;
                    if (rc31 >= 0 && rc31 <= span)
                        ring[(start + rc31) & rmask] =
                            make_int4(ws->bout[0][st & 31], ws->bout[1][st & 31], ws->bout[2][st & 31], 0);
                }
            }
            __syncwarp();
            const int cbase = (t - lane) & (CP_RING - 1);
            bool fin = false;
            std::integral_constant<bool, true> yes;
            std::integral_constant<bool, false> no;
            if (EAGER && MODE == MODE_INSPECT && top == 0 && t < 32) {
#pragma unroll 1
                for (int u = 0; u < 16; ++u)
                    if (step(yes, yes, t + u, u, u & 3, cbase)) { fin = true; break; }
            } else if (t + 15 <= span) {
                // steady state: no lane is past column N during these 16 steps (lanes still left of the strip's
                // first column compute dead cells: all their inputs are dead and their threshold is >= -(Y+1));
                // 4-step unrolled body keeps the hot loop inside the instruction cache
#pragma unroll 1
                for (int q = 0; q < 16 && !fin; q += 4) {
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        if (step(no, no, t + q + j, q + j, j, cbase)) { fin = true; break; }
                }
            } else {
#pragma unroll 1
                for (int u = 0; u < 16; ++u)
                    if (step(yes, no, t + u, u, u & 3, cbase)) { fin = true; break; }
            }
            if (fin) break;
            t += 16;
        }

        // ------------------------------------------------------------------ strip finish
        const int e = start + tfinal - 31;  // lane 31's last column
        __syncwarp();
        if (lane < 16) {  // park the last (partial) block's bottom rows in the ring
            const int st = t + lane, rc31 = st - 31;
            if (st <= tfinal && rc31 >= 0 && rc31 <= span)
                ring[(start + rc31) & rmask] =
                    make_int4(ws->bout[0][st & 31], ws->bout[1][st & 31], ws->bout[2][st & 31], 0);
        }
        if constexpr (MODE == MODE_EXEC) {
            if ((tfinal % SPW) != SPW - 1) io.codes[wbase + (long long)(tfinal / SPW) * 32 + lane] = cw;
        }
        cum_words += (long long)(tfinal / SPW + 1) * 32;
        if constexpr (MODE == MODE_INSPECT) {
            if (__any_sync(FULL, upd)) bound_words = cum_words;
            upd = false;
        }
        const int Wtail = ws->bout[2][tfinal & 31];
        if (e - start + 4 > rmask) {  // strip wider than the ring: the parked row has been overwritten
            flags |= SF_RING;
            break;
        }
        __syncwarp();
        // V of the boundary row beyond e: max of the old boundary and this strip's tail (exact, reading R3)
        for (int c = e + 1 + lane; c <= Emax; c += 32) {
            const int4 v = ring[c & rmask];
            ring[c & rmask] = make_int4(NEG, NEG, imax(v.z, Wtail), 0);
        }
        if (e >= Emax) {
            Emax = e;
            Wfar = Wtail;
        } else {
            Wfar = imax(Wfar, Wtail);
        }
        int first = INT_MAX, last = -1;
        for (int c0 = start; c0 <= e; c0 += 32) {
            const int c = c0 + lane;
            const bool lv = c <= e && ring[c & rmask].x != NEG;
            const unsigned bal = __ballot_sync(FULL, lv);
            if (bal) {
                if (first == INT_MAX) first = c0 + __ffs(bal) - 1;
                last = c0 + 31 - __clz(bal);
            }
        }
        __syncwarp();
        if (MODE == MODE_INSPECT) {
            // int32 range guard (reading R8)
            if (__any_sync(FULL, best + OE >= SCORE_LIMIT)) {
                flags |= SF_OVERFLOW;
                break;
            }
        }
        if (top + H > M || last < 0) break;  // matrix bottom reached, or no live cell: extension ends (R6)
        if (Emax + 4 - first > rmask) {      // boundary band wider than the ring
            flags |= SF_RING;
            break;
        }
        if (first > start) Wleft0 = ring[(first - 1) & rmask].z;
        lastlive = last;
        start = first;
        __syncwarp();
    }

    if constexpr (MODE == MODE_INSPECT) {
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
    }
    if constexpr (MODE == MODE_CENSUS) {
#pragma unroll
        for (int off = 16; off; off >>= 1) cells += __shfl_xor_sync(FULL, cells, off);
    }
    out.best = best;
    out.bi = bi;
    out.bj = bj;
    out.flags = flags;
    out.bound_words = bound_words;
    out.cells = cells;
    out.words = cum_words;
}

}  // namespace fz
