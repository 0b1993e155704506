// side.cuh -- the strip engine: one one-sided extension, strip by strip (see dp.cuh for the cell math).
//
// Two schedules of the same sweep:
//  * SOLO (warp per problem): one warp runs strips 0, 1, 2, ... of a side.
//  * PIPE (block per problem, long sides): the K warps of a CTA run strips s = w, w+K, w+2K, ... of ONE side
//    concurrently; strip s consumes strip s-1's bottom row through the shared boundary ring as soon as it is
//    flushed (progress flags in shared memory), so a long side advances K strips at a time.  Every
//    synchronisation point (strip start, boundary loads, termination, strip finish) waits only on strip s-1,
//    which is why the result is identical to SOLO (the cone rule of reading R3 is local).
//
// Modes:
//  MODE_INSPECT: score-only pass that finds the peak ("lightweight inspector"), records the 17x17 corner
//                codes during the first steps of strip 0 for eager traceback, and bounds the
//                executor's traceback storage (the executor's allocation is sized by the inspector).
//  MODE_EXEC:    the trimmed executor: the same DP restricted to [0,i*]x[0,j*] (exact, because the
//                cone rule only looks inside the rectangle), writing 4-bit codes to HBM in a step-major
//                layout: word (t / SPW) * 32 + lane of a strip holds lane's R rows for SPW steps, so each warp
//                store is one coalesced 128-byte line (P:180's consolidation, done in registers).
//  MODE_CENSUS:  counts explored cells (origin + cells with a live diagonal/up/left neighbour), the GCUPS
//                numerator; not on the timed path.
//
// Per-step data movement (the paper's register exchange, re-designed for sm_100a):
//  * lane l receives the bottom row (X, D, W) of lane l-1 with a ROTATING shuffle (src = l-1 mod 32); lane 0
//    then overwrites what lane 31 sent with the previous strip's boundary value for its column (one predicated
//    128-bit shared load straight into the shuffle results), and lane 31 parks its own bottom row in shared
//    staging (one predicated 128-bit store).  No per-step global memory access, no selects.
//  * every BLK = 32 steps (16 in PIPE) the warp moves 32 boundary values global ring -> shared staging (prefetched into
//    registers one block ahead) and 32 parked bottom-row values shared -> global ring, both coalesced; the
//    parked values also give the bottom row's first/last live column (next strip's start, termination test).
//  * termination: each lane keeps the last step at which one of its R cells was live; the strip is done at
//    column x (lane 31's) iff no lane has had a live cell since it processed x and the boundary row has no
//    live cell at or after x -- the unrolled form of the per-lane "done" chain (lane l is done at x iff its
//    cells are dead at x and lane l-1 is done at x).  Tested every 4 steps.
#pragma once
#include <type_traits>

#include "dp.cuh"

namespace fz {

enum { MODE_INSPECT = 0, MODE_EXEC = 1, MODE_CENSUS = 2 };

#ifndef STEADY_UNROLL
#define STEADY_UNROLL 8  // steps per unrolled steady-state body (8: one termination test per body; 16 overflows the I-cache)
#endif
#ifndef TERM_MASK
#define TERM_MASK 7  // termination test every TERM_MASK + 1 steps (u & TERM_MASK == TERM_MASK; t is a multiple of 8)
#endif
// steps per staging block (refill of boundary/profiles, park of the bottom row): BLK for SOLO; PIPE uses 16 so a
// consumer strip trails its producer by fewer columns (flush granularity + prefetch distance)
constexpr int BLK = 32;
constexpr int PIPE_SLOTS = 8;  // 2K slots for K = 4 warps: a slot is reused only after its consumer finished

struct WarpSmem {
    int co[CP_RING + BLK];  // column codes of the query side as substitution-table byte offsets (code * SubTab::CODE),
                            // ring over relative columns (+BLK mirrored)
    int4 bin[BLK];          // boundary row staging {X, D, W, -}: lane 0's input of the current block
    int4 bout[BLK];         // lane 31's bottom-row outputs {X, D, W, -} awaiting the global ring
    // N masks of the side's target / query copies (nullptr: no N); kept here rather than in registers so the
    // strip loop's register budget (72 = 7 CTAs per SM) is unchanged -- read only at strip set-up and staging
    const uint16_t* anm;
    const uint16_t* bnm;
};

// Block-per-problem (PIPE) shared state of one side.  Strip s owns slot s % PIPE_SLOTS.
struct PipeShared {
    volatile int sid[PIPE_SLOTS];    // strip id whose start/progress the slot currently describes
    volatile int start[PIPE_SLOTS];  // strip start column
    volatile int wleft[PIPE_SLOTS];  // W(top-1, start-1) of the strip
    volatile int prog[PIPE_SLOTS];   // last bottom-row column flushed to the ring
    volatile int first[PIPE_SLOTS];  // first live bottom-row column flushed so far (INT_MAX: none yet)
    volatile int last[PIPE_SLOTS];   // last live bottom-row column flushed so far
    volatile int done[PIPE_SLOTS];   // strip id whose finish (tail update, side state) is complete
    volatile int end_strip;          // strip that ended the side (INT_MAX while running)
    volatile int Emax, Wfar;         // boundary-ring state after the last finished strip
    volatile unsigned flags;
    volatile long long cum_words, bound_words;
    volatile int maxsw, bound_maxsw;
    int best[8], bi[8], bj[8];       // per-warp peaks for the final reduction
};

struct SideIO {
    const uint32_t* __restrict__ Apk;  // target side (rows), packed; A_k at position Aoff + k - 1
    int64_t Aoff;
    int M;                              // rows 0..M
    const uint32_t* __restrict__ Bpk;  // query side (columns)
    int64_t Boff;
    int Bmax;                           // real query length (bases beyond are never read)
    int N;                              // columns 0..N (N <= Bmax; the executor trims to j*)
    int4* __restrict__ ring;            // boundary ring (per warp in SOLO, per CTA in PIPE), rmask + 1 entries
    int rmask;
    WarpSmem* ws;                       // shared staging of this warp
    unsigned subtab;                    // shared address of the substitution table (dp.cuh, SUBTAB_*)
    uint8_t* ecodes;                    // shared: EAGER_W^2 eager codes (inspector)
    int eager_max;
    uint32_t* __restrict__ codes;       // executor: the side's code words
    int2* __restrict__ stab;            // executor: per strip {start column, word offset}
    int budget;                         // SOLO inspector: strips before escalation to PIPE (INT_MAX: none)
    PipeShared* ps;                     // PIPE: shared side state
    int wi, K;                          // PIPE: warp index in the CTA, warps per side
    int maxsw;                          // PIPE executor: words reserved per strip (from the inspector)
    long long wlim;                     // SOLO executor: words reserved for the side (stores beyond are dropped
                                        // and reported: the executor self-check)
    int xexp;                           // executor: X (= S - O - E) the inspector found at (M, N) = (i*, j*)
                                        // (INT_MIN: not checked -- the untrimmed ablation ends elsewhere)
};

struct SideOut {
    int best, bi, bj;        // peak in X space (score = best + O + E), ties: min i, min j
    uint32_t flags;
    long long bound_words;   // inspector: executor words up to the peak strip (compact layout)
    int bound_maxsw;         // inspector: max words of one strip up to the peak strip (block layout)
    long long cells;         // census: explored cells (warp total)
    long long words;         // all strips' words (inspector: the untrimmed executor's storage)
    int maxsw_all;           // widest strip over all strips
    int nstrips;             // strips run
    int checkfail;           // executor self-check: 1 = S(i*, j*) != inspector score or a store past the reservation
};

template <int R>
struct StripGeom {
    static constexpr int H = 32 * R;
    static constexpr int SPW = 8 / R;  // steps per 32-bit code word
};

// column code: query base 0..3, 5 for an N (NM: the batch has N masks), 4 outside [1, N] (the origin column and
// beyond the end)
template <bool NM>
__device__ __forceinline__ int query_code(const SideIO& io, int c) {
    if (c < 1 || c > io.N) return 4;
    if constexpr (NM) {
        if (n_at(io.ws->bnm, io.Boff + c - 1)) return 5;
    }
    return base_at(io.Bpk, io.Boff + c - 1);
}

template <bool NM>
__device__ __forceinline__ void cp_store(const SideIO& io, int rc, int code) {
    const int v = code * SubTab<NM>::CODE;
    const int idx = rc & (CP_RING - 1);
    io.ws->co[idx] = v;
    if (idx < BLK) io.ws->co[idx + CP_RING] = v;
}

// Boundary row value at column c: the ring holds exact entries up to column lim, beyond it the row is dead
// with W = Wfar (reading R3: V beyond the last scanned column).  PIPE reads bypass L1 (written by other warps).
template <bool PIPE>
__device__ __forceinline__ int4 boundary(const int4* __restrict__ ring, int rmask, int c, int lim, int Wfar) {
    if (c <= lim) return PIPE ? __ldcg(ring + (c & rmask)) : ring[c & rmask];
    return make_int4(NEG, NEG, Wfar, 0);
}

__device__ __forceinline__ void pipe_wait() { __nanosleep(100); }

// executor traceback code bit: cw += bit if a > b, as one ISETP (ALU pipe) + one predicated IMAD (FMA pipe; `one`
// is a runtime 1 so ptxas cannot turn it into an ALU-pipe IADD3).  The bits of a word never overlap, so the add
// is an OR.
__device__ __forceinline__ void code_bit_gt(uint32_t& cw, int a, int b, uint32_t bit, int one) {
    asm("{ .reg .pred p; setp.gt.s32 p, %1, %2; @p mad.lo.u32 %0, %3, %4, %0; }"
        : "+r"(cw) : "r"(a), "r"(b), "r"(bit), "r"(one));
}

template <int R, int MODE, bool EAGER, bool PIPE, bool NM>
__device__ __forceinline__ void run_side(const DevParams& P, const SideIO& io, SideOut& out) {
    constexpr int H = StripGeom<R>::H;
    constexpr int SPW = StripGeom<R>::SPW;
    constexpr int BK = PIPE ? 16 : BLK;
    const int lane = threadIdx.x & 31;
    const bool stager = BK == 32 || lane < BK;  // lanes that move one staging entry per block
    const int src = (lane + 31) & 31;
    const int M = io.M, N = io.N;
    const int E = P.E, OE = P.OE, mY = -P.Y, mE = -P.E, mOE = -P.OE;
    const int one = P.one, zero = P.zero;
    const int rmask = io.rmask;
    int4* __restrict__ ring = io.ring;
    WarpSmem* __restrict__ ws = io.ws;
    PipeShared* __restrict__ ps = io.ps;
    const bool is31 = lane == 31;
    const bool is0 = lane == 0;
    const unsigned sb_in = (unsigned)__cvta_generic_to_shared(&ws->bin[0]);
    const unsigned sb_out = (unsigned)__cvta_generic_to_shared(&ws->bout[0]);

    // W left of column 0 is V(i,-1) - Y = -inf; any value <= -Y gives the same thresholds (only the origin has
    // no finite neighbour, and it is live for any threshold <= 0).  -(Y+1) keeps the cells that lanes compute
    // before the strip's first column (ramp-up, left of column 0) dead, so ramp-up runs unchecked.
    const int Wout = -P.Y - 1;
    // SOLO side state (registers); PIPE keeps it in *ps
    int start = 0, Wleft0 = Wout, lastlive = -1, Emax = -1, Wfar = NEG, nfirst = INT_MAX;
    int best = NEG + 1, bi = INT_MAX, bj = INT_MAX;
    long long cum_words = 0, bound_words = 0, cells = 0;
    int maxsw = 0, bound_maxsw = 0, nstr = 0;
    uint32_t flags = 0;
    bool upd = false;
    bool bad = false;        // executor self-check
    int xcap = INT_MIN;      // executor: X at (M, N)

    for (int s = PIPE ? io.wi : 0;; s += PIPE ? io.K : 1) {
        const int slot = s % PIPE_SLOTS, pslot = (s + PIPE_SLOTS - 1) % PIPE_SLOTS;
        // ------------------------------------------------------------------ strip start
        if constexpr (PIPE) {
            if (s * H > M) goto side_done;  // strip s-1 holds row M and ends the side: never start past it
            if (s == 0) {
                start = 0;
                Wleft0 = Wout;
            } else {
                // wait until strip s-1 has flushed its first live bottom cell, or has finished
                for (;;) {
                    if (ps->end_strip < s) goto side_done;
                    if (ps->sid[pslot] == s - 1) {
                        const int f = ps->first[pslot];
                        if ((f != INT_MAX && ps->prog[pslot] >= f) || ps->done[pslot] == s - 1) break;
                    }
                    pipe_wait();
                }
                __threadfence_block();
                if (ps->end_strip < s) goto side_done;
                start = ps->first[pslot];
                const int sp = ps->start[pslot];
                Wleft0 = start > sp ? __ldcg(ring + ((start - 1) & rmask)).z : ps->wleft[pslot];
            }
            __syncwarp();
            if (lane == 0) {
                ps->start[slot] = start;
                ps->wleft[slot] = Wleft0;
                ps->first[slot] = INT_MAX;
                ps->last[slot] = -1;
                ps->prog[slot] = start - 1;
                __threadfence_block();
                ps->sid[slot] = s;
            }
        } else {
            if (s > 0) {
                if (io.budget != INT_MAX && s >= io.budget) {  // long side: hand over to the block kernel
                    flags |= SF_ESCALATE;
                    break;
                }
                if (nfirst > start) Wleft0 = ring[(nfirst - 1) & rmask].z;
                start = nfirst;
            }
        }
        const int top = s * H;

        // ------------------------------------------------------------------ strip set-up
        static_assert(R % 2 == 0, "rows per lane come in pairs (substitution table entries)");
        unsigned tb[R / 2];  // per row pair: shared address of this lane's replica of the pair's table entries
        int X[R], I[R], W[R];
        const int r0 = top + lane * R;
        int nvalid = M - r0 + 1;
        nvalid = nvalid < 0 ? 0 : (nvalid > R ? R : nvalid);
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const int r = r0 + k;
            int a = 0;
            if (r >= 1 && r <= M) a = (NM && n_at(io.ws->anm, io.Aoff + r - 1)) ? 4 : base_at(io.Apk, io.Aoff + r - 1);
            if (k % 2 == 0) tb[k / 2] = io.subtab + (unsigned)(a * SubTab<NM>::NB * SUBTAB_ENTRY) + (unsigned)((lane & 15) * 8);
            else tb[k / 2] += (unsigned)(a * SUBTAB_ENTRY);
            X[k] = NEG;
            I[k] = NEG;
            W[k] = (r <= M) ? Wleft0 : BIG;
        }
        int xdiag = (top == 0 && lane == 0) ? -OE : NEG;  // origin: H(0,0) = -OE + 0 + OE = 0
        int4 bq = make_int4(NEG, NEG, NEG, 0);  // this lane's bottom row (X, D, W) -> lane + 1 (lane 31: boundary)
        const int span = N - start;
        const int tlast = span + 31;
        const long long wbase = PIPE ? (long long)s * io.maxsw : cum_words;  // executor: strip's first word
        if constexpr (MODE == MODE_EXEC) {
            if (lane == 0) io.stab[s] = make_int2(start, (int)wbase);
        }
        // boundary source: SOLO -> ring up to Emax; PIPE -> ring up to strip s-1's progress, or (once it has
        // finished) up to the side's Emax
        int blim = Emax, bwf = Wfar;
        bool pdone = !PIPE || s == 0;
        auto pipe_sync = [&](int chi) {  // PIPE: make boundary columns <= chi readable
            if constexpr (PIPE) {
                if (s == 0) {
                    blim = -1;
                    bwf = NEG;
                    return;
                }
                if (!pdone) {
                    for (;;) {
                        if (ps->done[pslot] == s - 1) {
                            __threadfence_block();
                            pdone = true;
                            blim = ps->Emax;
                            bwf = ps->Wfar;
                            break;
                        }
                        const int pg = ps->prog[pslot];
                        if (pg >= chi) {
                            __threadfence_block();
                            blim = pg;
                            break;
                        }
                        pipe_wait();
                    }
                }
            }
        };
        pipe_sync(start + 2 * BK - 1);
        // staging: boundary and column profiles for relative columns [0, BK); prefetch the next BK
        int4 bpre = make_int4(NEG, NEG, bwf, 0);
        int qpre = 4;
        if (stager) {
            ws->bin[lane] = boundary<PIPE>(ring, rmask, start + lane, blim, bwf);
            cp_store<NM>(io, lane, query_code<NM>(io, start + lane));
            bpre = boundary<PIPE>(ring, rmask, start + BK + lane, blim, bwf);
            qpre = query_code<NM>(io, start + BK + lane);
        }
        __syncwarp();
        uint32_t cw = 0;
        int lastlive_t = -1;  // last 4-step group end at which this lane had a live cell (termination)
        int cacc = NEG;       // max X of this lane over the current 4-step group
        int Xp[R];            // inspector: X of the previous (even) step, peak-tested with the next step
        bool vp = false;
#pragma unroll
        for (int k = 0; k < R; ++k) Xp[k] = NEG;
        int tfinal = 0;
        int bfirst = INT_MAX, blast = -1;  // bottom row's first/last live column (from the parked values)
        if constexpr (PIPE) lastlive = s == 0 ? -1 : INT_MAX;  // unknown until strip s-1 has finished

        // park steps [st0, stmax] (at most BK) of lane 31's outputs in the ring; track live columns
        auto park = [&](int st0, int stmax) {
            const int st = st0 + lane, rc31 = st - 31;
            const bool ok = stager && st <= stmax && rc31 >= 0 && rc31 <= span;
            int xv = NEG;
            if (ok) {
                const int4 v = ws->bout[st & (BK - 1)];
                xv = v.x;
                ring[(start + rc31) & rmask] = v;
            }
            const unsigned bal = __ballot_sync(FULL, ok && xv != NEG);
            if (bal) {
                const int c0 = start + st0 - 31;  // column of lane 0's entry
                if (bfirst == INT_MAX) bfirst = c0 + __ffs(bal) - 1;
                blast = c0 + 31 - __clz(bal);
            }
            if constexpr (PIPE) {
                const unsigned okb = __ballot_sync(FULL, ok);
                if (okb) {
                    __threadfence_block();
                    if (lane == 0) {
                        const int c0 = start + st0 - 31;
                        ps->first[slot] = bfirst;
                        ps->last[slot] = blast;
                        ps->prog[slot] = c0 + 31 - __clz(okb);
                    }
                }
            }
        };

        // one wavefront step: lane computes column start + tt - lane.  Returns true when the strip is done.
        auto step = [&](auto chk, auto eag, const int tt, const int u, const int j, const int cbase,
                        const unsigned sgo, const unsigned sgi) -> bool {
            constexpr bool CHK = decltype(chk)::value;
            constexpr bool EG = decltype(eag)::value;
            const int rc = tt - lane;
            const bool valid = CHK ? (unsigned)rc <= (unsigned)span : true;
            int xu = __shfl_sync(FULL, bq.x, src);
            int du = __shfl_sync(FULL, bq.y, src);
            int wu = __shfl_sync(FULL, bq.z, src);
            // lane 0 replaces what lane 31 sent with the boundary row for its column (relative column tt)
            ld_shared3_if(is0, sgi + 16u * (unsigned)j, xu, du, wu);
            if (valid) {
                const int co = ws->co[cbase + u];
                int vs[R];
#pragma unroll
                for (int p = 0; p < R / 2; ++p) ld_shared2(fma_add(co, one, (int)tb[p]), vs[2 * p], vs[2 * p + 1]);
                int xd = xdiag;
                xdiag = xu;
#pragma unroll
                for (int k = 0; k < R; ++k) {
                    const int h = fma_add(vs[k], one, xd);  // X_diag + sub(a_i, b_j) + O + E
                    const int d = __viaddmax_s32(du, mE, xu);
                    const int iv = __viaddmax_s32(I[k], mE, X[k]);
                    int sr;
                    if constexpr (MODE == MODE_EXEC) {
                        // traceback code (P:178's 2 + 1 + 1 bits), executor format: bit 0 d > h, bit 1 iv > max(h, d)
                        // (S source: I if bit 1, else D if bit 0, else H -- reading R4's H > D > I), bit 2 d > xu
                        // (D extends: strictly better than opening, R4b), bit 3 iv > X_left (I extends)
                        const int mhd = imax(h, d);
                        sr = imax(mhd, iv);
                        const uint32_t sh = (uint32_t)((((j % SPW) * R) + k) * 4);
                        code_bit_gt(cw, d, h, 1u << sh, one);
                        code_bit_gt(cw, iv, mhd, 2u << sh, one);
                        code_bit_gt(cw, d, xu, 4u << sh, one);
                        code_bit_gt(cw, iv, X[k], 8u << sh, one);
                    } else {
                        sr = __vimax3_s32(h, d, iv);
                    }
                    // live iff S_raw >= thr = max(W_up, W_left) (reading R3); W = max(thr, S_raw - Y) equals
                    // max(thr, S_live - Y) because a dead cell has S_raw - Y < S_raw < thr.  thr comes from the
                    // row above and the previous column (ready before S), so the dependent chain after S is one
                    // ISETP + the FMA-pipe kill, and W (one VIADDMNMX from S) is off the chain (measured 637 ->
                    // 621 ms on C2 against W-first with the live test S >= W)
                    const int thr = imax(wu, W[k]);
                    const int xn = kill_fma(sr, thr, mOE, one, zero);
                    const int wn = __viaddmax_s32(sr, mY, thr);
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
                }
                bq.x = xu;
                bq.y = du;
                bq.z = wu;
#pragma unroll
                for (int k = 0; k < R; k += 2) cacc = __vimax3_s32(cacc, X[k], X[k + 1]);
            }
            if constexpr (MODE == MODE_INSPECT) {
                // peak (reading R5): tested every second step against the group maximum (a rare, warp-uniform
                // slow path then scans both steps' cells in column order; ties -> smaller row, columns only grow).
                // Re-scanning a cell is harmless: only a strictly better score or an equal one in a smaller row
                // moves the peak.
                const bool odd = (j & 1) != 0;
                if (!odd) {
#pragma unroll
                    for (int k = 0; k < R; ++k) Xp[k] = X[k];
                    vp = valid;
                }
                if (odd || (CHK && tt == tlast)) {
                    if (__any_sync(FULL, cacc >= best)) {
                        const int c = start + rc;
                        if (odd) {
#pragma unroll
                            for (int k = 0; k < R; ++k) {
                                const int r = r0 + k;
                                const bool better = vp && (Xp[k] > best || (Xp[k] == best && r < bi));
                                best = better ? Xp[k] : best;
                                bi = better ? r : bi;
                                bj = better ? c - 1 : bj;
                                upd |= better;
                            }
                        }
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
            }
            // lane 31 parks its bottom row
            st_shared4_if(is31, sgo + 16u * (unsigned)j, bq);
            if constexpr (MODE == MODE_EXEC) {
                if ((j % SPW) == SPW - 1) {  // j == tt mod 4 and SPW divides 4
                    const long long wl = (long long)(tt / SPW) * 32 + lane;
                    // never past the reservation (PIPE: the strip's stride, SOLO: the side's words)
                    if (PIPE ? wl < io.maxsw : wbase + wl < io.wlim) io.codes[wbase + wl] = cw;
                    else bad = true;
                    cw = 0;
                }
            }
            if (j == 3) {
                // liveness per 4-step group: live anywhere in the group -> the group's last step (conservative)
                lastlive_t = imax(lastlive_t, __viaddmin_s32(cacc, -NEG - 1, tt));
                cacc = NEG;
            }
            if (j == 3 && (u & TERM_MASK) == TERM_MASK && tt >= 31) {
                // done at lane 31's column x = start + tt - 31 iff every lane has been dead since it processed
                // x (step tt - 31 + lane) and the boundary row has no live cell at or after x
                const unsigned bal = __ballot_sync(FULL, lastlive_t < tt - 31 + lane);
                if (bal == FULL) {
                    if constexpr (PIPE) {
                        // deterministic (== SOLO): decide only once strip s-1 has either finished or flushed a
                        // live bottom cell at or after x; never on the timing of its progress
                        const int x = start + tt - 31;
                        while (lastlive == INT_MAX) {
                            if (ps->done[pslot] == s - 1) {
                                __threadfence_block();
                                lastlive = ps->last[pslot];
                                break;
                            }
                            if (ps->last[pslot] >= x) break;  // not done at x; lastlive stays unknown
                            pipe_wait();
                        }
                    }
                    if (start + tt - 31 > lastlive) {
                        tfinal = tt;
                        return true;
                    }
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
                park(t - BK, t - 1);
                pipe_sync(start + t + 2 * BK - 1);
                // staging refill for relative columns [t, t+BK) (prefetched), prefetch [t+BK, t+2BK)
                if (stager) {
                    const int rcn = t + lane;
                    ws->bin[rcn & (BK - 1)] = bpre;
                    cp_store<NM>(io, rcn, qpre);
                    bpre = boundary<PIPE>(ring, rmask, start + rcn + BK, blim, bwf);
                    qpre = query_code<NM>(io, start + rcn + BK);
                }
            }
            __syncwarp();
            const int cbase = (t - lane) & (CP_RING - 1);
            bool fin = false;
            std::integral_constant<bool, true> yes;
            std::integral_constant<bool, false> no;
            // staging addresses of a 4-step group starting at step g (g % 4 == 0): out and in entry g%BLK + j
            auto sgo_of = [&](int g) { return sb_out + 16u * (unsigned)(g & (BK - 1)); };
            auto sgi_of = [&](int g) { return sb_in + 16u * (unsigned)(g & (BK - 1)); };
            if (EAGER && MODE == MODE_INSPECT && top == 0 && t < 32) {
#pragma unroll 1
                for (int u = 0; u < BK; ++u) {
                    const int g = t + (u & ~3);
                    if (step(yes, yes, t + u, u, u & 3, cbase, sgo_of(g), sgi_of(g))) { fin = true; break; }
                }
            } else if (t + BK - 1 <= span) {
                // steady state: no lane is past column N during these BK steps (lanes still left of the strip's
                // first column compute dead cells: all their inputs are dead and their threshold is >= -(Y+1));
                // 4-step unrolled body keeps the hot loop inside the instruction cache
#pragma unroll 1
                for (int q = 0; q < BK && !fin; q += STEADY_UNROLL) {
#pragma unroll
                    for (int h = 0; h < STEADY_UNROLL; h += 4) {
                        const unsigned sgo = sgo_of(t + q + h), sgi = sgi_of(t + q + h);
#pragma unroll
                        for (int j = 0; j < 4; ++j)
                            if (step(no, no, t + q + h + j, q + h + j, j, cbase, sgo, sgi)) { fin = true; break; }
                        if (fin) break;
                    }
                }
            } else {
#pragma unroll 1
                for (int u = 0; u < BK; ++u) {
                    const int g = t + (u & ~3);
                    if (step(yes, no, t + u, u, u & 3, cbase, sgo_of(g), sgi_of(g))) { fin = true; break; }
                }
            }
            if (fin) break;
            t += BK;
        }

        // ------------------------------------------------------------------ strip finish
        const int e = start + tfinal - 31;  // lane 31's last column
        __syncwarp();
        park(t, tfinal);  // the last (partial) block's bottom rows
        if constexpr (MODE == MODE_EXEC) {
            if ((tfinal % SPW) != SPW - 1) {
                const long long wl = (long long)(tfinal / SPW) * 32 + lane;
                if (PIPE ? wl < io.maxsw : wbase + wl < io.wlim) io.codes[wbase + wl] = cw;
                else bad = true;
            }
        }
        const int Wtail = ws->bout[tfinal & (BK - 1)].z;
        const int sw = (tfinal / SPW + 1) * 32;
        const bool anyupd = __any_sync(FULL, upd);
        upd = false;
        if constexpr (PIPE) {  // the side state is sequential: wait for strip s-1's finish
            if (s > 0) {
                while (ps->done[pslot] != s - 1) pipe_wait();
                __threadfence_block();
            }
            Emax = ps->Emax;
            Wfar = ps->Wfar;
            cum_words = ps->cum_words;
            bound_words = ps->bound_words;
            maxsw = ps->maxsw;
            bound_maxsw = ps->bound_maxsw;
            flags = ps->flags;
        }
        if constexpr (MODE == MODE_INSPECT && !PIPE) {
        }
        if constexpr (MODE == MODE_EXEC) {
            // self-check input: the lane holding row M ends the strip with X(M, N) in its registers (the peak
            // (M, N) = (i*, j*) is live, so the strip cannot have stopped before that lane reached column N)
#pragma unroll
            for (int k = 0; k < R; ++k)
                if (r0 + k == M) xcap = X[k];
            if (__any_sync(FULL, bad)) flags |= SF_CHECKFAIL;
        }
        const int maxsw_prev = maxsw;
        cum_words += sw;
        maxsw = sw > maxsw ? sw : maxsw;
        if (MODE == MODE_INSPECT && anyupd) {
            // Storage of the trimmed executor, sized from the inspector ("allocate ... according to the
            // exact size needed"): the executor runs strips 0..s* = i*/H and its strip k covers columns
            // [start_k, j*] only, stopping no later than this strip did, i.e. min(tfinal, j* - start + 31) steps.
            // The bound is taken whenever a lane's peak moves: full widths for the strips above, the trimmed
            // width of this strip (with the warp's largest peak column, an upper bound of j*); exact for peaks in
            // the last strip with an update, an upper bound otherwise.
            int mbj = bj == INT_MAX ? 0 : bj;
#pragma unroll
            for (int off = 16; off; off >>= 1) mbj = imax(mbj, __shfl_xor_sync(FULL, mbj, off));
            const int sp = mbj - start > 0 ? mbj - start : 0;
            const int tt2 = tfinal < sp + 31 ? tfinal : sp + 31;
            const int tw = (tt2 / SPW + 1) * 32;
            // strips above: each also covers at most columns [0, j*] (start_k >= 0)
            const int wj = ((mbj + 31) / SPW + 1) * 32;
            const long long above = cum_words - sw;
            const long long cap = (long long)s * wj;
            bound_words = (above < cap ? above : cap) + tw;
            bound_maxsw = imax(maxsw_prev < wj ? maxsw_prev : wj, tw);
        }
        bool over = false;
        if (e - start + 4 > rmask) {  // strip wider than the ring: the parked row has been overwritten
            flags |= SF_RING;
            over = true;
        }
        if (!over) {
            __syncwarp();
            // V of the boundary row beyond e: max of the old boundary and this strip's tail (exact, reading R3)
            for (int c = e + 1 + lane; c <= Emax; c += 32) {
                const int4 v = PIPE ? __ldcg(ring + (c & rmask)) : ring[c & rmask];
                ring[c & rmask] = make_int4(NEG, NEG, imax(v.z, Wtail), 0);
            }
            if (e >= Emax) {
                Emax = e;
                Wfar = Wtail;
            } else {
                Wfar = imax(Wfar, Wtail);
            }
            if (MODE == MODE_INSPECT && __any_sync(FULL, best + OE >= SCORE_LIMIT)) {  // int32 guard (R8)
                flags |= SF_OVERFLOW;
                over = true;
            }
            if (top + H > M || blast < 0) over = true;  // matrix bottom, or no live cell: extension ends (R6)
            if (!over && Emax + 4 - bfirst > rmask) {   // boundary band wider than the ring
                flags |= SF_RING;
                over = true;
            }
        }
        __syncwarp();
        if constexpr (PIPE) {
            if (lane == 0) {
                ps->Emax = Emax;
                ps->Wfar = Wfar;
                ps->cum_words = cum_words;
                ps->bound_words = bound_words;
                ps->maxsw = maxsw;
                ps->bound_maxsw = bound_maxsw;
                ps->flags = flags;
                if (over) ps->end_strip = s;
                __threadfence_block();
                ps->done[slot] = s;
            }
            __syncwarp();
            if (over) break;
        } else {
            nstr = s + 1;
            if (over) break;
            lastlive = blast;
            nfirst = bfirst;
            __syncwarp();
        }
    }
side_done:
    if constexpr (MODE == MODE_EXEC) {  // X at (i*, j*) -> best (the PIPE block below takes the max over warps)
        best = xcap;
#pragma unroll
        for (int off = 16; off; off >>= 1) best = imax(best, __shfl_xor_sync(FULL, best, off));
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
    if constexpr (PIPE) {
        if (lane == 0) {
            ps->best[io.wi] = best;
            ps->bi[io.wi] = bi;
            ps->bj[io.wi] = bj;
        }
        __syncthreads();
        best = ps->best[0];
        bi = ps->bi[0];
        bj = ps->bj[0];
        for (int w = 1; w < io.K; ++w) {
            const int ob = ps->best[w], oi = ps->bi[w], oj = ps->bj[w];
            if (ob > best || (ob == best && (oi < bi || (oi == bi && oj < bj)))) {
                best = ob;
                bi = oi;
                bj = oj;
            }
        }
        flags = ps->flags;
        bound_words = ps->bound_words;
        bound_maxsw = ps->bound_maxsw;
        cum_words = ps->cum_words;
        maxsw = ps->maxsw;
        nstr = ps->end_strip + 1;
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
    out.bound_maxsw = bound_maxsw;
    out.cells = cells;
    out.words = cum_words;
    out.maxsw_all = maxsw;
    out.nstrips = nstr;
    // executor self-check: the recomputed S(i*, j*) equals the inspector's peak, no store left the reservation
    out.checkfail = (MODE == MODE_EXEC && ((flags & SF_CHECKFAIL) || (io.xexp != INT_MIN && best != io.xexp))) ? 1 : 0;
}

// Reset the block-per-problem shared state before a side (one thread; caller synchronises the CTA).
__device__ __forceinline__ void pipe_reset(PipeShared* ps) {
    for (int k = 0; k < PIPE_SLOTS; ++k) {
        ps->sid[k] = -1;
        ps->done[k] = -1;
        ps->first[k] = INT_MAX;
        ps->last[k] = -1;
        ps->prog[k] = -1;
    }
    ps->end_strip = INT_MAX;
    ps->Emax = -1;
    ps->Wfar = NEG;
    ps->flags = 0;
    ps->cum_words = 0;
    ps->bound_words = 0;
    ps->maxsw = 0;
    ps->bound_maxsw = 0;
}

}  // namespace fz
