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
#pragma once
#include "dp.cuh"

namespace fz {

enum { MODE_INSPECT = 0, MODE_EXEC = 1, MODE_CENSUS = 2 };

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
    int2* cpring;                       // shared: CP_RING + 16 column-profile entries
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

// Column profile ring refill: entry for relative column rc (column start + rc) at index rc & 127 (+ mirror).
__device__ __forceinline__ void cp_put(const SideIO& io, int start, int rc) {
    const int c = start + rc;
    int b = 4;
    if (c >= 1 && c <= io.N) b = base_at(io.Bpk, io.Boff + c - 1);
    const int2 v = io.cptab[b];
    const int idx = rc & (CP_RING - 1);
    io.cpring[idx] = v;
    if (idx < 16) io.cpring[idx + CP_RING] = v;
}

template <int R, int MODE, bool EAGER>
__device__ __forceinline__ void run_side(const DevParams& P, const SideIO& io, SideOut& out) {
    constexpr int H = StripGeom<R>::H;
    constexpr int SPW = StripGeom<R>::SPW;
    const int lane = threadIdx.x & 31;
    const int M = io.M, N = io.N;
    const int E = P.E, OE = P.OE, OEmY = P.OE - P.Y, mE = -P.E;
    const unsigned amask = lane == 0 ? 0u : (1u << (lane - 1));
    const int rmask = io.rmask;
    int4* __restrict__ ring = io.ring;

    int start = 0, Wleft0 = NEG, lastlive = -1, Emax = -1, Wfar = NEG;
    int best = NEG + 1, bi = INT_MAX, bj = INT_MAX;
    long long cum_words = 0, bound_words = 0, cells = 0;
    uint32_t flags = 0;
    bool upd = false;

    // row -1 lies outside the matrix: dead, V = -inf.  Two sentinel entries (lane 0 double-buffers).
    if (lane == 0) {
        ring[0] = make_int4(NEG, NEG, NEG, 0);
        ring[1] = make_int4(NEG, NEG, NEG, 0);
    }
    __syncwarp();

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
        const int lim2 = lane == 0 ? Emax + 2 : INT_MIN;
        const int t0l = lane == 0 ? lastlive - start : INT_MAX;
        int4 B0 = make_int4(NEG, NEG, NEG, 0), B1 = B0;
        if (lane == 0) {
            B0 = ring[start & rmask];
            B1 = ring[(start + 1) & rmask];
        }
        long long wbase = cum_words;  // executor: this strip's first word (relative to the side)
        if constexpr (MODE == MODE_EXEC) {
            if (lane == 0) io.stab[s] = make_int2(start, (int)wbase);
        }
        uint32_t cw = 0;
        unsigned prevb = 0;
        int tfinal = 0;

        cp_put(io, start, lane);  // relative columns [0, 32)
        __syncwarp();

        // one wavefront step: lane computes column start + tt - lane.  Returns true when the strip is done.
        auto step = [&](auto eag, const int tt, const int u, const int cbase, int4& BU) -> bool {
            constexpr bool EG = decltype(eag)::value;
            const int rc = tt - lane;
            const bool valid = (unsigned)rc <= (unsigned)span;
            int xu = __shfl_up_sync(FULL, xb, 1);
            int du = __shfl_up_sync(FULL, db, 1);
            int wu = __shfl_up_sync(FULL, wb, 1);
            if (lane == 0) {
                xu = BU.x;
                du = BU.y;
                wu = BU.z;
            }
            if (start + tt + 2 <= lim2) BU = ring[(start + tt + 2) & rmask];
            bool done = false;
            if (valid) {
                const int2 cp = io.cpring[cbase + u];
                int xd = xdiag;
                xdiag = xu;
                int cm = NEG;
#pragma unroll
                for (int k = 0; k < R; ++k) {
                    const int h = xd + prmt(cp.x, cp.y, sel[k]) + OE;
                    const int d = __viaddmax_s32(du, mE, xu);
                    const int iv = __viaddmax_s32(I[k], mE, X[k]);
                    const int sr = __vimax3_s32(h, d, iv);
                    const int thr = imax(wu, W[k]);
                    const int xn = (sr >= thr) ? sr - OE : NEG;
                    const int wn = __viaddmax_s32(xn, OEmY, thr);
                    if constexpr (MODE == MODE_EXEC) {
                        const uint32_t code = cell_code(h, d, iv, du, xu, I[k], X[k], E);
                        cw |= code << ((((tt % SPW) * R) + k) * 4);
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
                    cm = imax(cm, xn);
                }
                xb = xu;
                db = du;
                wb = wu;
                if constexpr (MODE == MODE_INSPECT) {
                    if (cm >= best) {
                        const int c = start + rc;
#pragma unroll
                        for (int k = 0; k < R; ++k) {
                            const int r = r0 + k;
                            if (X[k] > best || (X[k] == best && r < bi)) {
                                best = X[k];
                                bi = r;
                                bj = c;
                                upd = true;
                            }
                        }
                    }
                }
                if (lane == 31) ring[(start + rc) & rmask] = make_int4(xb, db, wb, 0);
                done = cm == NEG;
            }
            if constexpr (MODE == MODE_EXEC) {
                if ((tt % SPW) == SPW - 1) {
                    io.codes[wbase + (long long)(tt / SPW) * 32 + lane] = cw;
                    cw = 0;
                }
            }
            done = done && (((prevb & amask) != 0) || tt > t0l);
            prevb = __ballot_sync(FULL, done);
            if ((int)prevb < 0 || tt == tlast) {
                tfinal = tt;
                return true;
            }
            return false;
        };

        int t = 0;
        for (;;) {
            if (t > 0 && lane < 16) cp_put(io, start, t + 16 + lane);
            __syncwarp();
            const int cbase = (t - lane) & (CP_RING - 1);
            bool fin = false;
            if (EAGER && MODE == MODE_INSPECT && top == 0 && t < 32) {
                std::integral_constant<bool, true> eg;
#pragma unroll
                for (int u = 0; u < 16; u += 2) {
                    if (step(eg, t + u, u, cbase, B0)) { fin = true; break; }
                    if (step(eg, t + u + 1, u + 1, cbase, B1)) { fin = true; break; }
                }
            } else {
                std::integral_constant<bool, false> eg;
#pragma unroll
                for (int u = 0; u < 16; u += 2) {
                    if (step(eg, t + u, u, cbase, B0)) { fin = true; break; }
                    if (step(eg, t + u + 1, u + 1, cbase, B1)) { fin = true; break; }
                }
            }
            if (fin) break;
            t += 16;
        }

        // ------------------------------------------------------------------ strip finish
        const int e = start + tfinal - 31;  // lane 31's last column
        if constexpr (MODE == MODE_EXEC) {
            if ((tfinal % SPW) != SPW - 1) io.codes[wbase + (long long)(tfinal / SPW) * 32 + lane] = cw;
        }
        cum_words += (long long)(tfinal / SPW + 1) * 32;
        if constexpr (MODE == MODE_INSPECT) {
            if (__any_sync(FULL, upd)) bound_words = cum_words;
            upd = false;
        }
        const int Wtail = __shfl_sync(FULL, wb, 31);
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
        if (lane == 0) {
            ring[(Emax + 1) & rmask] = make_int4(NEG, NEG, Wfar, 0);
            ring[(Emax + 2) & rmask] = make_int4(NEG, NEG, Wfar, 0);
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
