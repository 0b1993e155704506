/* seed_oracle.c -- TEST INFRASTRUCTURE ONLY (never linked into the product; only tests/, smoke() and bench.py's
 * cpu_baseline leg may load it).  Plain CPU reference of the seeding + filtering stage that precedes the gapped
 * extension ("a lightweight exact-match search identifies short
 * sequences (19 base pairs long) to serve as seed sites ... the second stage filters the seed sites to obtain a
 * shorter list of promising seed sites ... the third stage extends the filtered seed sites").
 *
 * The paper fixes only the 19-bp seed span; the rest follows LASTZ's documented defaults [ext] and is listed
 * as readings S1-S6 in DESIGN.md:
 *   S1 spaced seed: a pattern of span L (default 19) with w care positions ('1'; default 12of19
 *      "1110100110010101111"); the word at position p is the codes A0 C1 G2 T3 at p + care offsets.
 *   S2 hit (t, q): the words at T[t..] and Q[q..] are equal, or (transitions on) differ at exactly one care
 *      position by a transition (A<->G, C<->T).
 *   S3 ungapped x-drop extension of a hit along its diagonal: right from (t, q) and left from (t-1, q-1); per
 *      direction the running sum of sub() is tracked, the extent is the shortest prefix reaching the first
 *      strict maximum (start value 0, extent 0) and the walk stops when the sum falls more than X below that
 *      maximum (s < best - X) or at a sequence end.  HSP = [t-l, t+r) x [q-l, q+r), score = best_l + best_r.
 *   S4 filter: keep an HSP iff score >= hspthresh.
 *   S5 identical HSPs (same t_start, q_start, length) are reported once.
 *   S6 anchor (the gapped extension's cut point): the HSP midpoint t_start + length/2, q_start + length/2.
 *      Output sorted by (anchor t, anchor q, t_start, length).
 *   S7 N (code 4): a word with an N at a care position matches nothing; in the walks any pair with an N scores
 *      n_score (reading R13).
 * Written for clarity: a sorted (word, position) index of T, a binary search per query word and variant, one
 * loop per extension.  No blocking, no fusion.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    int64_t t_start, q_start;
    int32_t length, score;
} fzs_hsp;

typedef struct {
    uint32_t key;
    int64_t pos;
} kp;

static int code_of(char c) {
    switch (c) {
        case 'A': case 'a': return 0;
        case 'C': case 'c': return 1;
        case 'G': case 'g': return 2;
        case 'T': case 't': return 3;
        case 'N': case 'n': return 4;
        default: return -1;
    }
}

static int cmp_kp(const void* a, const void* b) {
    const kp* x = (const kp*)a;
    const kp* y = (const kp*)b;
    if (x->key != y->key) return x->key < y->key ? -1 : 1;
    return x->pos < y->pos ? -1 : (x->pos > y->pos);
}

static int cmp_hsp_id(const void* a, const void* b) {
    const fzs_hsp* x = (const fzs_hsp*)a;
    const fzs_hsp* y = (const fzs_hsp*)b;
    if (x->t_start != y->t_start) return x->t_start < y->t_start ? -1 : 1;
    if (x->q_start != y->q_start) return x->q_start < y->q_start ? -1 : 1;
    return x->length < y->length ? -1 : (x->length > y->length);
}

static int cmp_hsp_anchor(const void* a, const void* b) {
    const fzs_hsp* x = (const fzs_hsp*)a;
    const fzs_hsp* y = (const fzs_hsp*)b;
    const int64_t xt = x->t_start + x->length / 2, yt = y->t_start + y->length / 2;
    const int64_t xq = x->q_start + x->length / 2, yq = y->q_start + y->length / 2;
    if (xt != yt) return xt < yt ? -1 : 1;
    if (xq != yq) return xq < yq ? -1 : 1;
    if (x->t_start != y->t_start) return x->t_start < y->t_start ? -1 : 1;
    return x->length < y->length ? -1 : (x->length > y->length);
}

/* S1: word at position p (care offsets off[0..w-1]), 2 bits per care position, first care position highest.
 * S7: *valid = 0 if a care position holds an N. */
static uint32_t word_at(const int8_t* s, int64_t p, const int* off, int w, int* valid) {
    uint32_t k = 0;
    *valid = 1;
    for (int c = 0; c < w; ++c) {
        if (s[p + off[c]] == 4) *valid = 0;
        k = (k << 2) | (uint32_t)(s[p + off[c]] & 3);
    }
    return k;
}

/* reading R13: any pair with an N scores n_score */
static int64_t subst(const int32_t* sub16, int32_t n_score, int a, int b) {
    return (a == 4 || b == 4) ? n_score : sub16[4 * a + b];
}

/* Returns 0, -1 (bad argument), -2 (bad base), -4 (out of memory), -6 (out buffer too small: *n_out = needed). */
int fzs_find(const char* T, int64_t tlen, const char* Q, int64_t qlen, const char* pattern, int transitions,
             const int32_t* sub16, int32_t n_score, int32_t xdrop, int32_t hspthresh, fzs_hsp* out, int64_t cap,
             int64_t* n_out, int64_t* n_hits) {
    const int L = (int)strlen(pattern);
    int off[32], w = 0;
    if (L < 1 || L > 64 || xdrop < 0) return -1;
    for (int i = 0; i < L; ++i) {
        if (pattern[i] == '1') {
            if (w == 16) return -1;
            off[w++] = i;
        } else if (pattern[i] != '0') {
            return -1;
        }
    }
    if (w < 1 || pattern[0] != '1' || pattern[L - 1] != '1') return -1;
    int8_t* t = (int8_t*)malloc((size_t)(tlen + 1));
    int8_t* q = (int8_t*)malloc((size_t)(qlen + 1));
    if (!t || !q) return -4;
    for (int64_t i = 0; i < tlen; ++i) if ((t[i] = (int8_t)code_of(T[i])) < 0) return -2;
    for (int64_t i = 0; i < qlen; ++i) if ((q[i] = (int8_t)code_of(Q[i])) < 0) return -2;

    /* index of T: (word, position) sorted */
    const int64_t nt = tlen >= L ? tlen - L + 1 : 0;
    kp* idx = (kp*)malloc(sizeof(kp) * (size_t)(nt + 1));
    int64_t ni = 0;
    for (int64_t p = 0; p < nt; ++p) {
        int valid;
        const uint32_t k = word_at(t, p, off, w, &valid);
        if (!valid) continue; /* S7 */
        idx[ni].key = k;
        idx[ni].pos = p;
        ++ni;
    }
    qsort(idx, (size_t)ni, sizeof(kp), cmp_kp);

    int64_t hcap = 1024, nh = 0, hits = 0;
    fzs_hsp* hs = (fzs_hsp*)malloc(sizeof(fzs_hsp) * (size_t)hcap);
    const int64_t nq = qlen >= L ? qlen - L + 1 : 0;
    for (int64_t qp = 0; qp < nq; ++qp) {
        int valid;
        const uint32_t k0 = word_at(q, qp, off, w, &valid);
        if (!valid) continue; /* S7 */
        const int nvar = transitions ? 1 + w : 1;
        for (int v = 0; v < nvar; ++v) {
            /* S2: variant 0 = exact word; variant 1 + c = transition at care position c (A<->G, C<->T: xor 2) */
            const uint32_t k = v == 0 ? k0 : k0 ^ (2u << (2 * (w - v)));
            /* binary search for the first index entry with this key */
            int64_t lo = 0, hi = ni;
            while (lo < hi) {
                const int64_t mid = (lo + hi) / 2;
                if (idx[mid].key < k) lo = mid + 1; else hi = mid;
            }
            for (int64_t e = lo; e < ni && idx[e].key == k; ++e) {
                const int64_t tp = idx[e].pos;
                ++hits;
                /* S3: right extension */
                int64_t s = 0, best_r = 0, r = 0;
                for (int64_t d = 0; tp + d < tlen && qp + d < qlen; ++d) {
                    s += subst(sub16, n_score, t[tp + d], q[qp + d]);
                    if (s > best_r) {
                        best_r = s;
                        r = d + 1;
                    }
                    if (s < best_r - xdrop) break;
                }
                /* S3: left extension */
                int64_t best_l = 0, l = 0;
                s = 0;
                for (int64_t d = 1; tp - d >= 0 && qp - d >= 0; ++d) {
                    s += subst(sub16, n_score, t[tp - d], q[qp - d]);
                    if (s > best_l) {
                        best_l = s;
                        l = d;
                    }
                    if (s < best_l - xdrop) break;
                }
                if (best_l + best_r >= hspthresh) { /* S4 */
                    if (nh == hcap) {
                        hcap *= 2;
                        hs = (fzs_hsp*)realloc(hs, sizeof(fzs_hsp) * (size_t)hcap);
                    }
                    hs[nh].t_start = tp - l;
                    hs[nh].q_start = qp - l;
                    hs[nh].length = (int32_t)(l + r);
                    hs[nh].score = (int32_t)(best_l + best_r);
                    ++nh;
                }
            }
        }
    }
    /* S5: identical HSPs once */
    qsort(hs, (size_t)nh, sizeof(fzs_hsp), cmp_hsp_id);
    int64_t nu = 0;
    for (int64_t i = 0; i < nh; ++i)
        if (nu == 0 || cmp_hsp_id(&hs[nu - 1], &hs[i]) != 0) hs[nu++] = hs[i];
    /* S6: anchor order */
    qsort(hs, (size_t)nu, sizeof(fzs_hsp), cmp_hsp_anchor);
    *n_out = nu;
    if (n_hits) *n_hits = hits;
    int rc = 0;
    if (nu > cap) rc = -6;
    else if (nu) memcpy(out, hs, sizeof(fzs_hsp) * (size_t)nu);
    free(hs);
    free(idx);
    free(t);
    free(q);
    return rc;
}
