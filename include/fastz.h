/*
 * fastz.h -- C ABI of the B200-native FastZ hot path (libfastz.so, ABI version 1).
 *
 * Batched gapped seed extension as in FastZ (Gundabolu, Vijaykumar, Thottethodi, SC'21; PAPER.md lines
 * cited as P:<n>): every seed (anchor) is extended by two one-sided affine-gap Gotoh alignments,
 * left and right of the cut point, explored under LASTZ-style y-drop pruning and
 * traced back from the highest-scoring cell.  The work runs in the paper's two stages: a
 * score-only inspector with eager 16x16 traceback, then a length-binned trimmed
 * executor that writes compact traceback bits, followed by traceback walks.
 * The exact semantics (cone reading of y-drop, tie rules, gap convention) are listed in DESIGN.md
 * "Readings" and are bit-identical to the CPU oracle in oracle/.
 *
 * Conventions (all entry points):
 *  - Return 0 (FASTZ_OK) or a negative fastz_status; fastz_strerror() describes it (thread-local detail).
 *  - The caller owns every buffer it passes in; the library copies what it needs before returning.
 *    The context owns its device memory (allocated through the optional dev_alloc hook or cudaMalloc).
 *  - One context per (device, stream) user; calls on one context are not thread-safe.
 *  - All device work is enqueued on the context's stream; fastz_extend_seeds synchronizes the stream
 *    twice (after binning, to size the traceback pool -- P:174 "allocation at kernel launch" -- and after
 *    the CIGAR length pass) and otherwise leaves results on the device.
 *  - Scores are int32.  A one-sided peak score >= 2^29 sets FASTZ_FLAG_OVERFLOW on that seed.
 *  - Self-check: the executor verifies that its recomputed S(i*,j*) equals the inspector's peak and that every
 *    traceback-code store stays inside the side's reservation; a failure returns FASTZ_ECUDA with the count.
 *
 * Environment knobs (experiments and tests; defaults are the measured best): FASTZ_R (rows per lane, 2 or 4;
 * default 4), FASTZ_INSPECT_ORDER=0 (take sides in seed order instead of predicted-longest first),
 * FASTZ_ESCALATE_STRIPS (hand sides longer than this many strips to the block-per-side inspector; default off),
 * FASTZ_BLOCK_BIN (smallest executor bin run block per side; default 3), FASTZ_POOL_MB (traceback-pool budget;
 * default 80% of free memory), FASTZ_RING_ENTRIES (boundary-ring entries per warp; wider bands take the wide
 * ring), FASTZ_L2_PERSIST=1 (boundary rings in an L2 persisting window during the inspector), FASTZ_SEED_HIT_CAP
 * (seeding scratch), FASTZ_TEST_SELFCHECK=1 (test hook: makes the executor self-check fail).
 * Packed inspector (two one-sided extensions per warp in 16-bit halves, results identical to the 32-bit
 * inspector): FASTZ_PAIR (0 never, 1 default: batches with >= 16 sides per warp slot and
 * parameters the 16-bit arithmetic holds, 2 always), FASTZ_PAIR_LONG (predicted bases from which a side runs in
 * the 32-bit inspector instead; default 32), FASTZ_PAIR_ESCAPE (strips after which a packed side is redone in
 * 32 bits; default 16, read at fastz_create), FASTZ_PAIR_DEBUG=1 (per-side and per-warp diagnostics to stderr).
 */
#ifndef FASTZ_H
#define FASTZ_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FASTZ_ABI_VERSION 1

typedef struct fastz_ctx fastz_ctx; /* opaque */

typedef enum {
    FASTZ_OK = 0,
    FASTZ_EINVAL = -1, /* bad argument or scoring parameter (ranges below) */
    FASTZ_EBASE = -2,  /* a sequence character outside ACGTNacgtn (index in fastz_strerror text) */
    FASTZ_ERANGE = -3, /* seed outside [0,len]; length >= 2^31; an explored band wider than the scratch */
    FASTZ_ENOMEM = -4, /* device allocation failed */
    FASTZ_ECUDA = -5,  /* CUDA runtime error (text in fastz_strerror) */
    FASTZ_ETRUNC = -6, /* output buffers too small: *n_out and *cigar_bytes hold the required sizes */
    FASTZ_ESTATE = -7  /* call out of order (e.g. get before extend) */
} fastz_status;

/*
 * Scoring (P:70-74 recurrences; P:108 y-drop).  Defaults (fastz_default_params) are LASTZ's documented
 * defaults -- the paper states none: HOXD70, O=400, E=30, Y=O+300E=9400, K=3000.
 *   sub[4*a+b]  substitution score, a = target base (DP row), b = query base (column), A0 C1 G2 T3;
 *               |sub| <= 32767.
 *   gap_open    O in [0, 2^24]; a gap of length k costs O + k*E (s_o + s_e).
 *   gap_extend  E in [1, 2^24].
 *   ydrop       Y in [0, 2^28]; a cell is pruned when its score is below max(V(i-1,j), V(i,j-1)) - Y, where
 *               V is the best score in the rectangle [0,i]x[0,j] (reading R3).
 *   gapped_threshold  K: only sets FASTZ_FLAG_ABOVE_K; never drops a seed.
 *   eager_max   eager-traceback window, 1..16 (16x16); sides whose peak has max(i*,j*) <= eager_max
 *               are traced back inside the inspector and skip the executor.
 *   n_score     N (unknown base, either case) in either sequence scores n_score against anything; default -100
 *               (reading R13; the paper is silent).  Spaced seeds never match across an N (S7).
 *   dev_alloc / dev_free / alloc_user  optional device allocator hooks (e.g. a framework caching
 *               allocator); NULL -> cudaMalloc / cudaFree.
 */
typedef struct {
    int32_t sub[16];
    int32_t gap_open;
    int32_t gap_extend;
    int32_t ydrop;
    int32_t gapped_threshold;
    int32_t eager_max;
    int32_t options;              /* FASTZ_OPT_* bits, 0 = the paper's full design (see below) */
    int32_t n_score;              /* score of any pair with an N (either sequence), |n_score| <= 32767 */
    int32_t reserved;
    void *(*dev_alloc)(size_t bytes, void *stream, void *user);
    void (*dev_free)(void *ptr, void *stream, void *user);
    void *alloc_user;
} fastz_params;

/* options: ablation switches mirroring the paper's Fig. 9 study and the downstream-output mode.
 * Results (scores, endpoints, CIGARs) are identical with any FASTZ_OPT_NO_* bit; only the work changes. */
#define FASTZ_OPT_NO_EAGER 1     /* no eager traceback: every side goes through the executor (P:166-170 off) */
#define FASTZ_OPT_NO_TRIM 2      /* executor recomputes the whole explored region, not [0,i*]x[0,j*] (P:172 off) */
#define FASTZ_OPT_NO_BINNING 4   /* one executor queue, warp per side, no length order (P:209-211 off) */
#define FASTZ_OPT_NO_BLOCK 8     /* no block-per-side scheduling of long sides (inspector and executor) */
#define FASTZ_OPT_TRACEBACK_ABOVE_K 16 /* traceback only seeds with score >= K; others get an empty CIGAR */
#define FASTZ_OPT_QUERY_REVCOMP 32 /* the context's query is the reverse complement of the `query` passed to
                                      fastz_create (minus strand, NEXT-4): seeds, HSPs and alignments use
                                      reverse-complement query coordinates; an invalid character is reported at
                                      its index in the caller's string */

/* A seed is a cut point: the right extension starts at T[tpos], Q[qpos]; the left one at T[tpos-1],
 * Q[qpos-1] going backwards.  0 <= tpos <= tlen, 0 <= qpos <= qlen. */
typedef struct {
    int64_t tpos, qpos;
} fastz_seed;

#define FASTZ_FLAG_ABOVE_K 1u   /* score >= gapped_threshold */
#define FASTZ_FLAG_LEFT_EAGER 2u  /* left side traced back eagerly in the inspector */
#define FASTZ_FLAG_RIGHT_EAGER 4u /* right side traced back eagerly */
#define FASTZ_FLAG_OVERFLOW 8u  /* a one-sided peak score reached 2^29 */
#define FASTZ_FLAG_NO_CIGAR 16u /* CIGAR skipped (FASTZ_OPT_TRACEBACK_ABOVE_K and score < K) */
#define FASTZ_FLAG_REDUNDANT 32u /* set by fastz_mark_redundant: dominated by another record (reading R14) */

/* One alignment per seed, in seed order (64 bytes). */
typedef struct {
    int32_t score;        /* left_score + right_score */
    int32_t left_score;   /* one-sided peak scores (>= 0: the cut point itself scores 0) */
    int32_t right_score;
    uint32_t flags;       /* FASTZ_FLAG_* */
    int64_t t_start, t_end; /* half-open, 0-based, forward strand: [tpos - i_L, tpos + i_R) */
    int64_t q_start, q_end; /* [qpos - j_L, qpos + j_R) */
    int64_t cigar_off;    /* offset of this seed's CIGAR text in the cigar buffer */
    int32_t cigar_len;    /* bytes, no terminator; "" for an empty alignment */
    int32_t reserved;
} fastz_alignment;

/* Fill *p with the defaults above.  Never fails. */
void fastz_default_params(fastz_params *p);

/*
 * Create a context on `device` using `cuda_stream` (a cudaStream_t; NULL -> the library creates its own
 * blocking stream, ordered after work on the legacy default stream).  Device inputs (sequences, seeds) must
 * be complete with respect to the context's stream when passed: a caller producing them on another stream
 * synchronizes it (or makes the context's stream wait on it) first.  `target`/`query` are ASCII (ACGTNacgtn) of tlen/qlen bytes, host or device memory
 * (detected with cudaPointerGetAttributes); they are copied, validated and packed to 2 bits per base
 * (forward and reversed copies) plus a 1-bit N mask on the device.  Errors: EINVAL (NULL pointers, bad params), ERANGE (a length
 * < 0 or >= 2^31), EBASE (invalid character), ENOMEM, ECUDA.  On error *out is NULL.
 */
int fastz_create(const fastz_params *p, const char *target, int64_t tlen, const char *query, int64_t qlen,
                 int device, void *cuda_stream, fastz_ctx **out);

/*
 * Packed input (multi-GPU broadcast of 2-bit sequences).  fastz_pack_sequence packs ASCII
 * (ACGTNacgtn; host or device memory) of `len` bases into caller-owned DEVICE buffers: words[(len+15)/16]
 * (16 bases per uint32, base k of a word in bits 2k+1:2k, A0 C1 G2 T3, an N packed as 0) and
 * nmask[(len+15)/16] (bit k of a uint16 = base k is N).  revcomp = 1 packs the reverse complement.
 * *has_n (may be NULL) = 1 if the sequence has an N.  Enqueued on `cuda_stream` (NULL = legacy default
 * stream); synchronizes it.  EBASE reports the first invalid character's index; EINVAL for host words/nmask.
 *
 * fastz_create_packed creates a context exactly like fastz_create from such device buffers (t_nmask /
 * q_nmask may be NULL: no N); the buffers are copied.  The context's query is the packed query as given
 * (pack with revcomp = 1 for the minus strand; FASTZ_OPT_QUERY_REVCOMP is not applied again).
 *
 * fastz_get_packed exposes a context's packed forward copies (which = 0 target, 1 query) as device pointers
 * valid until fastz_destroy (*nmask = NULL if the sequence has no N), e.g. as the source of a broadcast.
 */
int fastz_pack_sequence(const char *seq, int64_t len, int revcomp, uint32_t *words, uint16_t *nmask, int *has_n,
                        int device, void *cuda_stream);
int fastz_create_packed(const fastz_params *p, const uint32_t *t_words, const uint16_t *t_nmask, int64_t tlen,
                        const uint32_t *q_words, const uint16_t *q_nmask, int64_t qlen, int device,
                        void *cuda_stream, fastz_ctx **out);
int fastz_get_packed(fastz_ctx *c, int which, const uint32_t **words, const uint16_t **nmask, int64_t *len);

/*
 * Extend n seeds (host or device memory as `seeds_on_device` says; n may be 0).  Runs inspector, binning,
 * executor, traceback and CIGAR assembly on the context's stream; results stay on the device until
 * fastz_get_alignments.  Replaces the results of any previous call.  Errors: EINVAL, ERANGE (a seed out of
 * range -- index in fastz_strerror; the kernels treat such a seed as an empty extension and never read
 * outside the sequences, and the batch has no results), ENOMEM, ECUDA.
 */
int fastz_extend_seeds(fastz_ctx *c, const fastz_seed *seeds, int64_t n, int seeds_on_device);

/*
 * Copy the last batch's results to host memory: out[0..n) (n = seeds of the last extend call) and the
 * concatenated CIGAR text (SAM M/I/D, target = reference).  If out_cap < n or cigar_cap < total bytes,
 * nothing is copied, *n_out / *cigar_bytes receive the required sizes and FASTZ_ETRUNC is returned.
 * Synchronizes the stream.  ESTATE before any extend call.
 */
int fastz_get_alignments(fastz_ctx *c, fastz_alignment *out, int64_t out_cap, char *cigar, int64_t cigar_cap,
                         int64_t *n_out, int64_t *cigar_bytes);

/*
 * Device-resident view of the last batch (valid until the next extend/destroy): records and CIGAR text in
 * the context's device memory, for callers that keep results on the GPU (e.g. a NCCL gather).  The final
 * record/CIGAR writes are still queued on the context's stream when fastz_extend_seeds returns: a consumer on
 * another stream must synchronize the context's stream (or wait on an event recorded on it) before reading.
 */
int fastz_get_alignments_device(fastz_ctx *c, const fastz_alignment **recs, const char **cigar, int64_t *n,
                                int64_t *cigar_bytes);

/*
 * Per-side inspector results of the last batch, side index 2*s (left) and 2*s+1 (right) for seed s:
 * peak score, i* (target offset), j* (query offset) and side flags (bit 0 eager, bit 1 overflow).
 * Arrays of at least 2n entries (any may be NULL).  Synchronizes.  ESTATE before extend, ETRUNC if cap < 2n.
 */
int fastz_get_sides(fastz_ctx *c, int32_t *score, int32_t *ti, int32_t *qj, uint32_t *flags, int64_t cap);

/*
 * Explored-cell census of the last batch: re-runs the inspector's DP in a counting variant and writes the
 * number of explored cells of each side (the origin plus every cell with a live diagonal, upper or left
 * neighbour -- the GCUPS numerator) into cells[2n].  Not part of the extension; synchronizes.
 */
int fastz_census(fastz_ctx *c, int64_t *cells, int64_t cap);

/* Stage timings (ms, CUDA events on the stream) and work counts of the last extend call. */
typedef struct {
    float ms_total, ms_upload, ms_inspect, ms_bin, ms_execute, ms_traceback, ms_combine;
    int32_t n_warp_slots;
    int64_t n_seeds, n_sides, n_eager_sides, n_exec_sides;
    int64_t bin_counts[8];        /* per side: bin 0 = eager (<=16), 1 <=512, 2 <=2048, 3 <=8192, 4 <=32768,
                                     5 <=131072, 6 larger (4x rule) */
    int64_t exec_words;           /* 32-bit traceback-code words written by the executor */
    int64_t cigar_bytes;
    int64_t n_launches;           /* kernels of this library launched by the call (CUB scans excluded) */
    int64_t n_waves;              /* executor/traceback waves under the traceback-pool budget */
    int64_t n_escalated;          /* sides handed from the warp inspector to the block inspector */
    int64_t n_wide_sides;         /* sides whose explored band outgrew the regular boundary ring and ran with the
                                     wide ring (very large Y or indel-rich long alignments) */
    int64_t exec_reserved_words;  /* traceback-pool words reserved for the executor (>= exec_words) */
    int64_t n_selfcheck_fail;     /* executor self-check failures: S(i*,j*) != inspector score, or code words
                                     outside a side's reservation (always 0; nonzero -> FASTZ_ECUDA) */
    int64_t n_packed_sides;       /* sides given to the packed (two per warp, 16-bit) inspector */
    int64_t n_long_sides;         /* sides predicted long, inspected first by the 32-bit inspector */
    int64_t n_redo_sides;         /* packed sides that reached the 16-bit value cap and were re-inspected in 32 bits
                                     (results never depend on which inspector ran a side) */
} fastz_stats;
int fastz_get_stats(fastz_ctx *c, fastz_stats *s);

/*
 * Seeding + ungapped filter (the stage before the gapped extension).  PAPER.md P:93:
 * "a lightweight exact-match search identifies short sequences (19 base pairs long) to serve as seed sites
 * ... the second stage filters the seed sites to obtain a shorter list of promising seed sites ... the third
 * stage extends the filtered seed sites".  The paper fixes only the 19-bp span; the defaults are LASTZ's
 * [ext] and the exact semantics are readings S1-S6 of DESIGN.md:
 *   pattern     spaced seed over '0'/'1', NUL-terminated, span 1..32, 1..16 care positions ('1'), first and
 *               last character '1'; default "1110100110010101111" (12of19).  A hit (t, q) needs the target
 *               and query words (bases at the care positions) to be equal -- S1/S2.
 *   transitions 1: additionally allow one transition (A<->G, C<->T) at one care position (default 1) -- S2.
 *   xdrop       X >= 0 of the ungapped x-drop walk right of and left of each hit along its diagonal; a walk
 *               stops when its running score falls more than X below its maximum (default 910) -- S3.
 *   hspthresh   an HSP (the two walks' best extents) is kept iff its score >= hspthresh (default 3000) -- S4.
 * Scores use the context's sub[] matrix.
 */
typedef struct {
    char pattern[64];
    int32_t transitions;
    int32_t xdrop;
    int32_t hspthresh;
    int32_t reserved;
} fastz_seed_params;

/* An HSP: the ungapped segment T[t_start, t_start+length) x Q[q_start, q_start+length) and its score. */
typedef struct {
    int64_t t_start, q_start;
    int32_t length, score;
} fastz_hsp;

void fastz_default_seed_params(fastz_seed_params *sp);

/*
 * Find the HSPs between the context's target and query (forward strands) on the device: spaced-seed hits,
 * ungapped x-drop filter, identical HSPs reported once (S5), sorted by anchor (S6).  `hsps` (may be NULL)
 * receives the HSPs and `anchors` (may be NULL) their cut points for fastz_extend_seeds: the HSP midpoint
 * (t_start + length/2, q_start + length/2).  Both are host buffers of `cap` entries; if cap is too small,
 * nothing is copied, *n_out holds the required count and FASTZ_ETRUNC is returned.  *n_hits (may be NULL)
 * receives the number of raw seed hits.  Synchronizes the stream.  Errors: EINVAL (bad pattern/params),
 * ERANGE (a single query word with more hits than device memory holds), ENOMEM, ECUDA.
 */
int fastz_find_hsps(fastz_ctx *c, const fastz_seed_params *sp, fastz_hsp *hsps, fastz_seed *anchors, int64_t cap,
                    int64_t *n_out, int64_t *n_hits);

/*
 * Redundant-alignment post-pass.  PAPER.md P:110: LASTZ "terminates an ongoing seed
 * extension upon reaching a previously-discovered alignment"; that skip is sequential-order dependent,
 * so FastZ extends every seed.  This call applies it after the fact, order-free (reading R14), on the
 * last batch's device records: among records with FASTZ_FLAG_ABOVE_K, record b dominates record a (a != b) iff
 * b.t_start <= a.t_start, a.t_end <= b.t_end, b.q_start <= a.q_start, a.q_end <= b.q_end, b.score >= a.score,
 * and (the boxes differ, or b.score > a.score, or b's seed index is lower).  A dominated record is redundant:
 * FASTZ_FLAG_REDUNDANT is set in its device record (a later fastz_get_alignments returns it; the bit is
 * recomputed, not accumulated, on every call) and, if `redundant` (host, may be NULL) is given, redundant[s] =
 * 1, else 0, for every seed s (cap >= n, else FASTZ_ETRUNC and nothing is written).  *n_redundant (may be
 * NULL) receives the count.  Records below K are never marked.  Synchronizes the stream.  ESTATE before any
 * extend call; ENOMEM / ECUDA as elsewhere.
 */
int fastz_mark_redundant(fastz_ctx *c, uint8_t *redundant, int64_t cap, int64_t *n_redundant);

/*
 * The same post-pass (reading R14) on any caller-owned record set, without a context -- e.g. the records of
 * several batches or ranks gathered in one array (paper_conf_sc_gundaboluvt21_b200/dist.py).  recs[n] holds
 * fastz_alignment records (host memory if recs_on_device == 0, else device memory of `device`); only score,
 * flags, t_start/t_end and q_start/q_end are read, and FASTZ_FLAG_REDUNDANT is recomputed in place in every
 * record's flags.  The seed index of the tie rule is the record's position in the array; coordinates must lie
 * in [0, 2^31) as fastz_extend_seeds produces them.  redundant (host,
 * may be NULL) receives n marks, *n_redundant (may be NULL) the count.  Uses a private stream and scratch
 * device memory (cudaMalloc), freed before returning; synchronous.  EINVAL (n < 0, n >= 2^31, recs NULL with
 * n > 0), ENOMEM, ECUDA.
 */
int fastz_mark_redundant_records(fastz_alignment *recs, int64_t n, int recs_on_device, uint8_t *redundant,
                                 int64_t *n_redundant, int device);

/* Release everything; NULL-safe. */
void fastz_destroy(fastz_ctx *c);

/* Static text for a status code, plus the detail of the last error on this thread. */
const char *fastz_strerror(int status);

/* INT32 peak microbenchmark (roofline denominator): runs independent integer max/add chains on every SM
 * for ~`ms` milliseconds on `device` and reports integer lane-operations per second. */
int fastz_int_peak(int device, float ms, double *ops_per_s, double *sm_clock_mhz);

#ifdef __cplusplus
}
#endif
#endif /* FASTZ_H */
