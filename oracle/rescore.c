/*
 * rescore.c -- TEST INFRASTRUCTURE ONLY (like everything under oracle/): an independent re-scoring check
 * of finished alignment records, usable on whole batches at any size.
 *
 * Only tests/ may load it.  It shares no code with the product and does not run the DP: it only re-adds
 * the scores of the operations a CIGAR spells out, from the definitions the paper fixes:
 *   - an alignment column of two bases scores sub(a, b) (reading R13: a pair with an N scores
 *     n_score);
 *   - a gap of length k costs O + k*E (s_o + s_e on the first gap base, s_e on every further one);
 *   - a seed's alignment is its left one-sided alignment followed by its right one, each with its
 *     own gap opens (SURVEY c.8): a gap run that crosses the cut point (tpos, qpos) pays O on both sides.
 *
 * For every record it checks: the CIGAR is well formed ("<len><op>" runs, len >= 1, op in M/I/D, no two
 * adjacent runs with the same op -- the text merges them, c.8); the path starts at (t_start, q_start),
 * passes exactly through the cut point and ends at (t_end, q_end); the left and right parts re-score to
 * left_score and right_score; score = left_score + right_score.  A record flagged "no CIGAR" (FASTZ flag 16)
 * is skipped.
 */
#include <stdint.h>
#include <string.h>

typedef struct {                 /* fastz_alignment (include/fastz.h), 64 bytes; restated here, not included */
    int32_t score, left_score, right_score;
    uint32_t flags;
    int64_t t_start, t_end, q_start, q_end;
    int64_t cigar_off;
    int32_t cigar_len, reserved;
} fzr_record;

static int code(char c) {
    switch (c) {
        case 'A': case 'a': return 0;
        case 'C': case 'c': return 1;
        case 'G': case 'g': return 2;
        case 'T': case 't': return 3;
        default: return 4;   /* N */
    }
}

/* returns 0 if record r passes, else a positive reason code */
static int check_one(const char *T, int64_t tlen, const char *Q, int64_t qlen, int64_t tpos, int64_t qpos,
                     const fzr_record *r, const char *cig, const int32_t *sub, int32_t O, int32_t E,
                     int32_t n_score, int64_t *got_left, int64_t *got_right) {
    *got_left = *got_right = 0;
    if (r->flags & 16u) return 0;
    if (r->t_start < 0 || r->t_start > tpos || r->t_end < tpos || r->t_end > tlen) return 1;
    if (r->q_start < 0 || r->q_start > qpos || r->q_end < qpos || r->q_end > qlen) return 1;
    if ((int64_t)r->score != (int64_t)r->left_score + (int64_t)r->right_score) return 2;
    int64_t t = r->t_start, q = r->q_start;
    int64_t score[2] = {0, 0};
    int side = (t == tpos && q == qpos) ? 1 : 0;   /* 0 = left of the cut, 1 = right */
    char prev[2] = {0, 0};                        /* previous op of each side (gap opens) */
    char last_run = 0;
    int64_t k = 0;
    const int64_t n = r->cigar_len;
    while (k < n) {
        int64_t len = 0;
        int digits = 0;
        while (k < n && cig[k] >= '0' && cig[k] <= '9') {
            len = len * 10 + (cig[k] - '0');
            ++k;
            ++digits;
            if (len > ((int64_t)1 << 40)) return 3;
        }
        if (k >= n || digits == 0 || len < 1) return 3;
        const char op = cig[k++];
        if (op != 'M' && op != 'I' && op != 'D') return 3;
        if (op == last_run) return 3;             /* adjacent equal runs must have been merged */
        last_run = op;
        for (int64_t s = 0; s < len; ++s) {
            if (op == 'M') {
                if (t >= tlen || q >= qlen) return 4;
                const int a = code(T[t]), b = code(Q[q]);
                score[side] += (a == 4 || b == 4) ? n_score : sub[4 * a + b];
                ++t;
                ++q;
            } else if (op == 'D') {                /* target base against a gap */
                if (t >= tlen) return 4;
                score[side] -= (prev[side] == 'D') ? E : (int64_t)O + E;
                ++t;
            } else {                               /* query base against a gap */
                if (q >= qlen) return 4;
                score[side] -= (prev[side] == 'I') ? E : (int64_t)O + E;
                ++q;
            }
            prev[side] = op;
            if (side == 0) {
                if (t == tpos && q == qpos) side = 1;
                else if (t > tpos || q > qpos) return 5;   /* stepped past the cut point */
            }
        }
    }
    if (side == 0 && !(t == tpos && q == qpos)) return 5;
    if (t != r->t_end || q != r->q_end) return 6;
    *got_left = score[0];
    *got_right = score[1];
    if (score[0] != r->left_score || score[1] != r->right_score) return 7;
    return 0;
}

/*
 * Check n records.  seeds: n (tpos, qpos) int64 pairs; recs: n fzr_record; cigar: the concatenated text.
 * reason[s] (if not NULL) receives the per-record result (0 = ok).  Returns the number of failing records;
 * *first_bad = index of the first failure (-1 if none).
 */
int64_t fzr_rescore(const char *T, int64_t tlen, const char *Q, int64_t qlen, const int64_t *seeds, int64_t n,
                    const void *recs, const char *cigar, int64_t cigar_bytes, const int32_t *sub, int32_t O,
                    int32_t E, int32_t n_score, int32_t *reason, int64_t *first_bad) {
    const fzr_record *R = (const fzr_record *)recs;
    int64_t nbad = 0;
    *first_bad = -1;
    for (int64_t s = 0; s < n; ++s) {
        int rc;
        int64_t gl, gr;
        if (R[s].cigar_off < 0 || R[s].cigar_len < 0 || R[s].cigar_off + R[s].cigar_len > cigar_bytes) rc = 8;
        else rc = check_one(T, tlen, Q, qlen, seeds[2 * s], seeds[2 * s + 1], &R[s], cigar + R[s].cigar_off, sub, O,
                            E, n_score, &gl, &gr);
        if (reason) reason[s] = rc;
        if (rc) {
            if (*first_bad < 0) *first_bad = s;
            ++nbad;
        }
    }
    return nbad;
}
