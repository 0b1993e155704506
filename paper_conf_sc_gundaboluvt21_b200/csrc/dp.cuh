// dp.cuh -- the warp-strip y-drop DP shared by the inspector, the executor and the census (sm_100a).
//
// One warp computes one one-sided extension ("a single seed extension DP task to a warp").  The
// DP matrix (rows i = target side A_1..A_M, columns j = query side B_1..B_N) is cut into horizontal
// strips of H = 32*R rows; lane l owns R consecutive rows of the strip and holds their S/I/V state in
// registers (the paper's cyclic use-and-discard buffers, re-designed: registers per ROW, not
// per diagonal).  The warp sweeps the strip's columns as a skewed wavefront (lane l lags l columns, the
// anti-diagonal layout of P:124 realised in time rather than in memory); each step every lane updates its
// R cells of one column and hands its bottom row (X, D, W) to lane l+1 with three SHFLs ("register
// exchange").  Only the strip's last row leaves the registers: lane 31 streams it to a per-warp ring in
// global memory (L2-resident) and lane 0 of the next strip reads it back ("boundary cells ... written
// out to memory to be re-loaded later for the next strip").
//
// Arithmetic: X = S - (O+E) is carried instead of S, so the gap opens of the cell below
// and to the right are single VIADDMNMX ops:  D = max(D_up - E, X_up),  I = max(I_left - E, X_left),
// H = X_diag + sub + (O+E),  S = max3(H, D, I).  y-drop uses W = V - Y (V = best live score of the
// rectangle [0,i]x[0,j], reading R3):  thr = max(W_up, W_left), live iff S >= thr, W = max(thr, S - Y).
// Only S is killed (dead X = NEG); I and D keep their values -- by the lemma in DESIGN.md (V never decreases
// along a predecessor edge) this yields the same live set, scores, peak and on-path traceback codes as
// killing all three.  Substitution scores (with O+E folded in) come from a shared-memory table indexed by the
// column's query code (streamed through a per-warp ring as a byte offset) and the lane's row-pair bases: one
// conflict-free LDS.64 per row pair and step, no ALU-pipe select.
#pragma once
#include <cstdint>
#include <climits>

namespace fz {

constexpr int NEG = -(1 << 30);   // dead score (X space)
constexpr int BIG = (1 << 30);    // threshold of rows beyond M: nothing there is ever live
constexpr unsigned FULL = 0xffffffffu;
constexpr int SCORE_LIMIT = 1 << 29;
constexpr int CP_RING = 128;      // column-profile ring entries per warp (+BLK mirrored)
constexpr int EAGER_W = 17;       // eager code window: rows/cols 0..16 (16x16)
// Substitution table in shared memory: entry e = code * NB^2 + a0 * NB + a1 (query code: A C G T = 0..3, 4 = the
// origin column (sub = 0), 5 = N; target bases of a row pair a0, a1, 4 = N) holds int2
// {sub(a0, code) + O + E, sub(a1, code) + O + E}, replicated 16x so that the 16 lanes of a half-warp read 16
// distinct bank pairs (conflict-free LDS.64).  NB = 4 (codes 0..4) for batches without N -- the layout and
// instruction stream of the N-free path are unchanged -- and NB = 5 (codes 0..5) when a sequence has an N
// (reading R13: any pair with an N scores n_score).
constexpr int SUBTAB_REP = 16;
constexpr int SUBTAB_ENTRY = SUBTAB_REP * 8;    // bytes per entry
template <bool NM>
struct SubTab {
    static constexpr int NB = NM ? 5 : 4;                  // target-base symbols per row
    static constexpr int CODE = NB * NB * SUBTAB_ENTRY;    // bytes per query code
    static constexpr int NCODES = NM ? 6 : 5;
    static constexpr int INTS = NCODES * CODE / 4;
};
constexpr int SUBTAB_INTS = SubTab<true>::INTS;  // shared allocation (the larger layout)

// side flags
constexpr uint32_t SF_EAGER = 1u, SF_OVERFLOW = 2u, SF_RING = 4u, SF_ESCALATE = 8u, SF_NOTB = 16u;
constexpr uint32_t SF_WIDE = 32u;  // inspected with the wide ring (band wider than the regular ring)
constexpr uint32_t SF_CHECKFAIL = 64u;  // executor self-check failed (S(i*, j*) mismatch or a store past the reservation)
constexpr uint32_t SF_PAIR = 1u << 20;  // inspected by the packed kernel (pair.cuh); k_eager clears it after the eager walk
constexpr int OPT_NO_EAGER = 1, OPT_NO_TRIM = 2, OPT_NO_BINNING = 4, OPT_NO_BLOCK = 8, OPT_TB_ABOVE_K = 16;
constexpr int OPT_SELFCHECK_TEST = 1 << 20;  // internal (FASTZ_TEST_SELFCHECK): expect S(i*,j*) + 1, so the check fires

struct DevParams {
    int sv[30];        // sv[5 * code + a] = score(a, code) + O + E: code 0..3 query base, 4 origin column (0), 5 N;
                       // target base a 0..3, 4 = N (reading R13: any pair with an N scores n_score)
    int O, E, Y, OE;   // gap open, extend, y-drop, O+E
    int K, eager_max;
    int one, zero;     // runtime 1 and 0: keep adds/selects as IMAD on the FMA pipe (ALU pipe is the limiter)
    int options;       // FASTZ_OPT_* (fastz.h)
};

// d = a * one + c on the FMA pipe (one == 1 at run time; ptxas cannot fold it into an ALU IADD3)
__device__ __forceinline__ int fma_add(int a, int one, int c) {
    int d;
    asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(c));
    return d;
}

// y-drop kill (reading R3) with the select on the FMA pipe: x = (s >= thr) ? s - OE : NEG
__device__ __forceinline__ int kill_fma(int s, int thr, int mOE, int one, int zero) {
    int x = fma_add(s, one, mOE);
    // x * zero + NEG depends on x, so ptxas cannot hoist it into a SEL on the ALU pipe
    asm("{ .reg .pred p; setp.lt.s32 p, %1, %2; @p mad.lo.s32 %0, %0, %3, %4; }"
        : "+r"(x) : "r"(s), "r"(thr), "r"(zero), "n"(NEG));
    return x;
}

// 64-bit shared load of two words
__device__ __forceinline__ void ld_shared2(int addr, int& x, int& y) {
    asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(addr));
}

// predicated shared-memory store / load (keeps per-lane staging as predicated instructions, not a branch)
__device__ __forceinline__ void st_shared_if(bool p, unsigned addr, int v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q st.shared.b32 [%1], %2; }" ::"r"((unsigned)p), "r"(addr),
                 "r"(v));
}
__device__ __forceinline__ void ld_shared_if(bool p, unsigned addr, int& v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %1, 0; @q ld.shared.b32 %0, [%2]; }" : "+r"(v) : "r"((unsigned)p), "r"(addr));
}

// predicated 128-bit shared store / load of a register quad (x, y, z, w)
__device__ __forceinline__ void st_shared4_if(bool p, unsigned addr, int4 v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q st.shared.v4.b32 [%1], {%2, %3, %4, %5}; }" ::"r"((unsigned)p),
                 "r"(addr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w));
}
__device__ __forceinline__ void ld_shared4_if(bool p, unsigned addr, int4& v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %4, 0; @q ld.shared.v4.b32 {%0, %1, %2, %3}, [%5]; }"
                 : "+r"(v.x), "+r"(v.y), "+r"(v.z), "+r"(v.w)
                 : "r"((unsigned)p), "r"(addr));
}

// predicated 128-bit shared load into three fresh registers (4th word discarded)
__device__ __forceinline__ void ld_shared3_if(bool p, unsigned addr, int& x, int& y, int& z) {
    int pad;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %4, 0; @q ld.shared.v4.b32 {%0, %1, %2, %3}, [%5]; }"
                 : "+r"(x), "+r"(y), "+r"(z), "=r"(pad)
                 : "r"((unsigned)p), "r"(addr));
}

__device__ __forceinline__ int prmt(int a, int b, int s) {
    int d;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(s));
    return d;
}

// base k (0-based position pos) of a 2-bit packed sequence (16 bases per word, base 0 in bits 1:0)
__device__ __forceinline__ int base_at(const uint32_t* __restrict__ pk, int64_t pos) {
    return (int)((__ldg(pk + (pos >> 4)) >> ((pos & 15) * 2)) & 3u);
}

// N mask: bit (pos & 15) of 16-bit word pos >> 4 (nullptr: the sequence has no N)
__device__ __forceinline__ bool n_at(const uint16_t* __restrict__ nm, int64_t pos) {
    return nm != nullptr && ((__ldg(nm + (pos >> 4)) >> (pos & 15)) & 1u);
}

__device__ __forceinline__ int imax(int a, int b) { return a > b ? a : b; }

// Traceback code of a cell (2 bits S source + 1 bit D extends + 1 bit I extends).
//   src 0 = H (diagonal), 1 = D (up), 2 = I (left); priority H > D > I (reading R4).
__device__ __forceinline__ uint32_t cell_code(int h, int d, int i, int du, int xu, int il, int xl, int E) {
    uint32_t src = d > h ? 1u : 0u;
    const int m = imax(h, d);
    src = i > m ? 2u : src;
    const uint32_t dext = (du - E) > xu ? 4u : 0u;
    const uint32_t iext = (il - E) > xl ? 8u : 0u;
    return src | dext | iext;
}

}  // namespace fz
