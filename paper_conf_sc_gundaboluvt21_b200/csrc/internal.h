// internal.h -- launchers shared between kernels.cu and api.cu (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include "dp.cuh"

namespace fz {

constexpr int WARPS = 4;  // warps per block of the persistent DP kernels

// Per-side arrays written by the inspector (index 2*seed + right).
struct SideArrays {
    int* score;          // peak score (S space)
    int* ti;             // i*
    int* qj;             // j*
    uint32_t* flags;     // SF_* | eager op count << 8
    unsigned long long* eops;  // eager ops, 2 bits each, emission order (peak -> origin)
    long long* bound;    // executor words bound, compact layout (0 for eager sides)
    int* maxsw;          // executor words of the widest strip up to the peak strip (block layout)
    int* nstrip;         // executor strips (i*/H + 1; all inspected strips under FASTZ_OPT_NO_TRIM)
};

struct Batch {
    const uint32_t *Tf, *Tr, *Qf, *Qr;  // packed target/query, forward and reversed
    const uint16_t *TfN, *TrN, *QfN, *QrN;  // their N masks (nullptr when the sequence has no N)
    int tlen, qlen;
    const long long* seeds;             // (tpos, qpos) pairs
    int nseeds;
};

struct ExecPlan {
    // per side (2n), exclusive scans in side order
    long long* woff;     // code-word offset of the side in the pool
    long long* soff;     // strip-table offset
    long long* roff;     // run-buffer offset
    int* bin;            // per side bin (0 = eager)
    int* list;           // executor order: non-eager sides, larger bins first; bins >= 3 (block per side)
                         // occupy list[0, totals[4])
    int* counters;       // [0] inspector queue, [1] executor warp queue, [2..8] bin counts, [10..16] bin cursors,
                         // [20] ring overflow, [21] escalated sides, [22] block inspector queue,
                         // [23] executor block queue, [24] wide (ring-overflow) sides, [28] predicted-long sides
                         // (32-bit inspector), [30] packed-inspector redo sides
    long long* totals;   // [0] words, [1] strips, [2] runs, [3] n_exec, [4] n_exec_block
    int* esc;            // escalated sides (inspector -> block inspector)
    long long* wl;       // executor words in list order (scratch)
    long long* wlo;      // exclusive scan of wl: pool offset of list position i
    int* wide;           // sides whose band overflowed the regular ring (counters[24] of them)
    int* redo;           // sides the packed inspector abandoned (value cap), re-inspected in 32 bits (counters[30])
};

struct Outputs {
    uint32_t* codes;     // executor pool
    int2* stab;          // strip tables
    uint32_t* runs;      // traceback runs (len << 2 | op), emission order
    int* nruns;          // per side
    long long* cig_len;  // per seed CIGAR length, then exclusive-scanned in place into offsets
    char* cigar;
    void* recs;          // fastz_alignment[n]
};

// Packed inspector constants (pair.cuh): stored 16-bit value = true value + Z
struct PairParams {
    unsigned Z;      // bias: stored = true + Z
    unsigned NEGb;   // dead X (and D / I never fall below it)
    unsigned BIGb;   // threshold of rows beyond M and columns beyond N: nothing there is live
    unsigned mE2;    // per-half (-E) mod 2^16
    unsigned mY2;    // -(Y * 0x10001): 32-bit add, no borrow since every S >= NEG_b >= Y
    unsigned mOE2;   // -(OE * 0x10001)
    unsigned limX;   // value cap: a half whose peak X (stored) reaches limX is redone in 32 bits
    int WoutT;       // W left of column 0 (true value, -(Y+1))
    int esc_strips;  // a packed side still running after this many strips is redone in 32 bits (long sides must
                     // not run packed: a lone packed warp steps ~2x slower than a 32-bit one)
    int2* hist;      // per warp slot and half: {start column, last step} of strips 0..PAIR_HIST-1 of the current
                     // side, for the exact executor reservation (nullptr: the 32-bit kernel's bound)
};

constexpr int PAIR_HIST = 16;
int pick_R();  // rows per lane (FASTZ_R env: 2, 4 or 8; default 4)

cudaError_t launch_pack(const char* src, int64_t n, uint32_t* fwd, uint32_t* rev, uint16_t* fwdn, uint16_t* revn,
                        long long* bad, int revcomp, cudaStream_t st);
cudaError_t launch_reverse_packed(const uint32_t* fwd, const uint16_t* fwdn, int64_t n, uint32_t* rev, uint16_t* revn,
                                  int* has_n, cudaStream_t st);
cudaError_t launch_validate_seeds(const long long* seeds, int n, int tlen, int qlen, long long* bad,
                                  cudaStream_t st);
int inspector_blocks_per_sm(int R);
// inspector order: predicted side lengths (ungapped walk) sorted longest first into order[nsides]
size_t order_tmp_bytes(int n);
cudaError_t launch_order(const Batch& b, const DevParams& P, int nsides, unsigned* keys_in, unsigned* keys_out,
                         int* vals_in, int* order, void* tmp, size_t tmp_bytes, cudaStream_t st);
// slist/nlist: inspect the nlist listed sides in that order (nullptr: all 2n sides in index order)
cudaError_t launch_inspect(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                           const SideArrays& sa, const ExecPlan& pl, int budget, const int* slist, int nlist,
                           cudaStream_t st);
// packed inspection (kernels.cu k_inspect_mixed): order[0, n1) in its 32-bit path (queue counters[35]; n1 = 0 when
// a concurrent k_inspect takes the predicted-long head order[0, nlong)), order[nlong, nsides) packed two per warp
// (queue counters[32]), and the sides the packed phase abandons (pl.redo, pre-set to -1; pushes counters[30],
// claims counters[34]) in its 32-bit path.  dbg: optional diagnostics buffer (FASTZ_PAIR_DEBUG).
int mixed_blocks_per_sm();
cudaError_t launch_inspect_mixed(int grid, const DevParams& P, const PairParams& Q, const Batch& b, int4* ring,
                                 int rmask, const SideArrays& sa, const ExecPlan& pl, const int* order, int nsides,
                                 int nlong, int n1, int budget, long long* dbg, cudaStream_t st);
// *count = number of sorted (descending) prediction keys >= thr: the sides the 32-bit inspector takes first
cudaError_t launch_split(const unsigned* keys_desc, int n, unsigned thr, int* count, cudaStream_t st);
// eager walk of the packed inspector's sides whose peak lies in the 17x17 corner; clears SF_PAIR
cudaError_t launch_eager(const DevParams& P, const Batch& b, const SideArrays& sa, int nsides, cudaStream_t st);
cudaError_t launch_inspect_block(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                                 const SideArrays& sa, const ExecPlan& pl, cudaStream_t st);
int escalate_strips();  // FASTZ_ESCALATE_STRIPS (default 16; 0 disables block-per-side inspection)
cudaError_t launch_census(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                          long long* cells, int* counter, const int* slist, int nlist, cudaStream_t st);
cudaError_t launch_bin(int R, const DevParams& P, const SideArrays& sa, int nsides, const ExecPlan& pl, void* scan_tmp,
                       size_t scan_tmp_bytes, long long* tmp_a, long long* tmp_b, long long* tmp_c,
                       cudaStream_t st);
size_t scan_tmp_bytes(int n);
// LPT order of the block-per-side executor sides list[0, nblock) (descending words), offsets recomputed
size_t lpt_tmp_bytes(int n);
cudaError_t launch_lpt(const ExecPlan& pl, int nblock, int nexec, const long long* words, long long* keys_in,
                       long long* keys_out, int* vals_in, void* sort_tmp, size_t sort_tmp_bytes, void* scan_tmp,
                       size_t scan_tmp_bytes, cudaStream_t st);
// flag the listed sides SF_WIDE (after their re-inspection with the wide ring)
cudaError_t launch_mark_wide(const SideArrays& sa, const int* list, int n, cudaStream_t st);
// list the sides flagged SF_WIDE (any order) and count them
cudaError_t launch_wide_list(const SideArrays& sa, int nsides, int* list, int* count, cudaStream_t st);
// redundant-alignment post-pass (dedup.cu; NEXT-3, reading R14)
size_t redundant_tmp_bytes(int n);
cudaError_t launch_redundant(void* recs, int n, void* tmp, size_t tmp_bytes, uint32_t* k1, uint32_t* k2, int* i1,
                             int* i2, int4* box, int2* sc, unsigned char* red, int* counters, cudaStream_t st);
cudaError_t launch_execute(int R, int grid, const DevParams& P, const Batch& b, int4* ring, int rmask,
                           const SideArrays& sa, const ExecPlan& pl, int lo, int hi, int nblock, long long base,
                           const Outputs& o, int wide, cudaStream_t st);
cudaError_t launch_traceback(int R, const SideArrays& sa, const ExecPlan& pl, int lo, int hi, int nblock,
                             long long base, const Outputs& o, cudaStream_t st);
cudaError_t launch_combine_len(const DevParams& P, const Batch& b, const SideArrays& sa, const ExecPlan& pl,
                               const Outputs& o, void* scan_tmp, size_t scan_tmp_bytes, long long* total,
                               cudaStream_t st);
cudaError_t launch_combine_write(const DevParams& P, const Batch& b, const SideArrays& sa,
                                 const ExecPlan& pl, const Outputs& o, cudaStream_t st);
cudaError_t int_peak_run(int device, float ms, double* ops_per_s, double* mhz);


// ---------------------------------------------------------------------------------------- seeding (seeds.cu)
struct SeedPattern {
    int L, w;      // span, care positions (1..16)
    int off[16];   // care offsets, ascending
    unsigned caremask;  // bit o set for every care offset o
};
struct UngappedParams {
    int sub[25];   // sub[5a+b], a = target code, b = query code, 4 = N (reading R13: n_score)
    int xdrop, hspthresh;
};
struct HspOut {    // layout of fastz_hsp
    long long t_start, q_start;
    int length, score;
};
size_t seed_sort_tmp_bytes(long long n);
cudaError_t seed_keys(const uint32_t* Tf, const uint16_t* TfN, long long nt, const SeedPattern& sp, uint32_t* keys,
                      int* pos, unsigned char* valid, cudaStream_t st);
cudaError_t seed_compact(void* tmp, size_t tmp_bytes, const uint32_t* kin, const int* pin, const unsigned char* valid,
                         long long nt, uint32_t* kout, int* pout, int* nsel, cudaStream_t st);
cudaError_t seed_sort_words(void* tmp, size_t tmp_bytes, const uint32_t* kin, uint32_t* kout, const int* vin,
                            int* vout, long long n, int bits, cudaStream_t st);
cudaError_t seed_bucket_start(const uint32_t* skeys, long long nt, int* start, long long nkeys, cudaStream_t st);
cudaError_t seed_count(const uint32_t* Qf, const uint16_t* QfN, long long q0, long long nq, const SeedPattern& sp, int nvar,
                       const uint32_t* skeys, const int* spos, const int* start, long long nt, long long* cnt,
                       long long* off, void* tmp, size_t tmp_bytes, cudaStream_t st);
cudaError_t seed_write_extend(const uint32_t* Tf, const uint32_t* Qf, const uint16_t* TfN, const uint16_t* QfN, int tlen, int qlen, long long q0, long long nq,
                              const SeedPattern& sp, int nvar, const uint32_t* skeys, const int* spos,
                              const int* start, long long nt, const long long* off, long long nh, int2* hits,
                              const UngappedParams& up, int4* hsp, unsigned char* keep, cudaStream_t st);
cudaError_t seed_select(void* tmp, size_t tmp_bytes, const int4* hsp, const unsigned char* keep, long long nh,
                        int4* out, int* nsel, cudaStream_t st);
// k1: n keys, k2: 2n keys, i1/i2: n ints; the final order is left in i1
cudaError_t seed_finish_sort(void* tmp, size_t tmp_bytes, const int4* hs, long long n, unsigned long long* k1,
                             unsigned long long* k2, int* i1, int* i2, cudaStream_t st);
cudaError_t seed_unique_emit(void* tmp, size_t tmp_bytes, const int4* hs, const int* order, long long n, int* flag,
                             int* pos, HspOut* out, long long* anchors, cudaStream_t st);

}  // namespace fz
