/*
 * fastz_oracle.c -- PLAIN, SLOW, OBVIOUSLY-CORRECT CPU ORACLE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  The product path (paper_conf_sc_gundaboluvt21_b200/) never does, and this file
 * shares no code, header, table or constant generator with it.
 *
 * What it computes (FastZ, Gundabolu/Vijaykumar/Thottethodi SC'21, /root/reference/PAPER.md, cited as
 * "P:<line>"):  LASTZ-style gapped seed extension.  Every seed is extended by two independent one-sided
 * alignments, left and right of the cut point, which are then added.  Each one-sided alignment
 * is the affine-gap Gotoh recurrence of Fig. 1, global at the cut point and free at the far
 * end ("ydrop_one_sided_align"), explored under y-drop pruning and traced back from
 * the highest-scoring cell using 1+1+2 traceback bits per cell.
 *
 * Readings of the paper that this oracle fixes (listed in DESIGN.md, "Readings"):
 *   R1 gap of length k costs O + k*E (s_o + s_e on open, s_e per extension).
 *   R2 no zero floor; S(0,0)=0, I(0,0)=D(0,0)=-inf (one-sided extension).
 *   R3 y-drop "cone" rule: V(i,j) = max of S over LIVE cells of the rectangle [0,i]x[0,j]; cell (i,j) is
 *      live iff S_raw(i,j) >= max(V(i-1,j), V(i,j-1)) - Y ("previously-completed scores along the row or
 *      column"; threshold relative to highest observed score).  Dead cells hold -inf.
 *   R4 source priority H > D > I; a gap extends only if strictly better than opening.
 *   R5 peak = max S over live cells; ties -> smallest i, then smallest j (row-major first).
 *   R6 extension ends at the first row without a live cell ("if all the scores of a row fall below").
 *   R7 explored cells (the GCUPS numerator) = origin + cells with a live diagonal/up/left predecessor.
 *   R8 peak scores >= 2^29 are flagged (score range of the int32 ABI), not an error of the method.
 *   R13 N (code 4, either sequence) scores n_score against anything; other non-ACGT characters are errors.
 *
 * Plain row-major scan; int64 arithmetic; one byte per traceback code (bits 1:0 = S source 0 H/1 D/2 I,
 * bit 2 = D extends, bit 3 = I extends -- P:178's 2+1+1 bits).  V(i-1, j) is obtained from a per-column
 * running maximum of live S (Vcol) so that V is exact even beyond the columns the previous row scanned.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#define NEG (-(INT64_C(1) << 60))
#define SCORE_LIMIT (INT64_C(1) << 29)

typedef struct {
    int32_t sub[16];          /* sub[4*a+b]: a = target base (row), b = query base (column); A0 C1 G2 T3 */
    int32_t gap_open;         /* O >= 0 */
    int32_t gap_extend;       /* E >= 1 */
    int32_t ydrop;            /* Y >= 0 */
    int32_t gapped_threshold; /* K: flag bit only */
    int32_t eager_max;        /* eager window: classification only */
    int32_t n_score;          /* reading R13: any pair with an N (code 4) scores n_score */
} fzo_params;

/* substitution score of target code a against query code b (A0 C1 G2 T3, N4; reading R13) */
static int64_t subst(const fzo_params *p, int a, int b) {
    return (a == 4 || b == 4) ? p->n_score : p->sub[4 * a + b];
}

typedef struct {
    int64_t score, i, j;   /* peak */
    int64_t explored;      /* R7 */
    int64_t rows;          /* last row holding a live cell, plus one */
    int64_t nops;          /* traceback ops written (origin-outward order) */
    int32_t overflow;      /* R8 */
    int32_t pad;
} fzo_side;

typedef struct {
    int64_t score, left_score, right_score;
    int64_t t_start, t_end, q_start, q_end;
    int64_t li, lj, ri, rj;
    int64_t l_explored, r_explored;
    int64_t cigar_off, cigar_len;
    int32_t flags, pad;    /* 1: score >= K, 2: left eager, 4: right eager, 8: overflow */
} fzo_alignment;

static inline int64_t max2(int64_t a, int64_t b) { return a > b ? a : b; }

/* growable workspace, one per thread */
typedef struct {
    uint8_t *codes; int64_t codes_cap;          /* codes of all scanned cells, row after row */
    int64_t *row_lo, *row_off; int64_t rows_cap; /* per row: first scanned column, offset into codes */
    int64_t *Vcol, *pS, *pD, *cS, *cD, *cI; int64_t cols_cap;  /* indexed by absolute column */
    int64_t vcol_dirty;                         /* Vcol[0 .. vcol_dirty) may hold values of a previous call */
    char *ops; int64_t ops_cap;
} fzo_ws;

static int ws_cols(fzo_ws *w, int64_t need) {
    if (need <= w->cols_cap) return 0;
    int64_t cap = w->cols_cap ? w->cols_cap : 1024;
    while (cap < need) cap *= 2;
    int64_t **arrs[6] = {&w->Vcol, &w->pS, &w->pD, &w->cS, &w->cD, &w->cI};
    for (int a = 0; a < 6; a++) {
        int64_t *p = (int64_t *)realloc(*arrs[a], (size_t)cap * sizeof(int64_t));
        if (!p) return -1;
        for (int64_t c = w->cols_cap; c < cap; c++) p[c] = NEG;
        *arrs[a] = p;
    }
    w->cols_cap = cap;
    return 0;
}
static int ws_rows(fzo_ws *w, int64_t need) {
    if (need <= w->rows_cap) return 0;
    int64_t cap = w->rows_cap ? w->rows_cap : 1024;
    while (cap < need) cap *= 2;
    int64_t *a = (int64_t *)realloc(w->row_lo, (size_t)cap * sizeof(int64_t));
    if (!a) return -1;
    w->row_lo = a;
    a = (int64_t *)realloc(w->row_off, (size_t)cap * sizeof(int64_t));
    if (!a) return -1;
    w->row_off = a;
    w->rows_cap = cap;
    return 0;
}
static int ws_codes(fzo_ws *w, int64_t need) {
    if (need <= w->codes_cap) return 0;
    int64_t cap = w->codes_cap ? w->codes_cap : 65536;
    while (cap < need) cap *= 2;
    uint8_t *p = (uint8_t *)realloc(w->codes, (size_t)cap);
    if (!p) return -1;
    w->codes = p; w->codes_cap = cap;
    return 0;
}
static int ws_ops(fzo_ws *w, int64_t need) {
    if (need <= w->ops_cap) return 0;
    int64_t cap = w->ops_cap ? w->ops_cap : 4096;
    while (cap < need) cap *= 2;
    char *p = (char *)realloc(w->ops, (size_t)cap);
    if (!p) return -1;
    w->ops = p; w->ops_cap = cap;
    return 0;
}
static void ws_free(fzo_ws *w) {
    free(w->codes); free(w->row_lo); free(w->row_off);
    free(w->Vcol); free(w->pS); free(w->pD); free(w->cS); free(w->cD); free(w->cI); free(w->ops);
    memset(w, 0, sizeof(*w));
}

/*
 * One-sided extension.  A[k-1] is A_k (rows, target side), B[k-1] is B_k (columns, query
 * side), both as codes 0..3.  On return w->ops[0 .. out->nops) holds the alignment ops 'M' 'I' 'D' in
 * origin-outward order.  Returns 0, or -1 on allocation failure.
 */
static int one_sided(const uint8_t *A, int64_t M, const uint8_t *B, int64_t N, const fzo_params *p,
                     fzo_side *out, fzo_ws *w) {
    const int64_t O = p->gap_open, E = p->gap_extend, Y = p->ydrop;
    memset(out, 0, sizeof(*out));
    if (ws_cols(w, 2) || ws_rows(w, 1)) return -1;
    for (int64_t c = 0; c < w->vcol_dirty; c++) w->Vcol[c] = NEG;  /* V(-1, .) = -inf */
    w->vcol_dirty = 0;

    int64_t best = 0, bi = 0, bj = 0;      /* the origin is live with S = 0 (R2, R5) */
    int64_t explored = 0, codes_used = 0;
    int64_t plo = 0, phi = -1;              /* previous row scanned range (none for row 0) */
    int64_t pfirst = -1, plast = -1;        /* previous row first/last live column */
    int64_t Vbase = NEG, vbase_upto = 0;    /* max of Vcol over columns < vbase_upto (frozen) */
    int64_t rows = 0;

    for (int64_t i = 0; i <= M; i++) {
        int64_t lo;
        if (i == 0) lo = 0;
        else {
            if (pfirst < 0) break;          /* R6: previous row had no live cell */
            lo = pfirst;
        }
        /* fold the frozen columns [vbase_upto, lo) into Vbase: no later row has a live cell there */
        for (int64_t c = vbase_upto; c < lo; c++) Vbase = max2(Vbase, w->Vcol[c]);
        if (lo > vbase_upto) vbase_upto = lo;

        if (ws_rows(w, i + 1)) return -1;
        w->row_lo[i] = lo;
        w->row_off[i] = codes_used;

        int64_t vup = Vbase;    /* V(i-1, j): running max of Vcol_{i-1} over [lo, j] with Vbase */
        int64_t vleft = Vbase;  /* V(i, j-1) */
        if (i == 0) { vup = NEG; vleft = NEG; }
        int64_t Sl = NEG, Il = NEG;  /* S(i, j-1), I(i, j-1): dead left of lo (or outside) */
        int live_l = 0;
        int64_t first = -1, last = -1;
        int64_t j = lo;
        for (;; j++) {
            if (j > N) break;
            if (i == 0) { if (j > 0 && !live_l) break; }
            else if (j > plast + 1 && !live_l) break;
            if (ws_cols(w, j + 2)) return -1;
            if (ws_codes(w, codes_used + 1)) return -1;

            /* predecessors (stored, post-kill values) */
            int64_t Su = NEG, Du = NEG, Sd = NEG;
            if (i >= 1 && j >= plo && j <= phi) { Su = w->pS[j]; Du = w->pD[j]; }
            if (i >= 1 && j >= 1 && j - 1 >= plo && j - 1 <= phi) Sd = w->pS[j - 1];
            int live_u = Su != NEG, live_d = Sd != NEG;
            if ((i == 0 && j == 0) || live_d || live_u || live_l) explored++;

            int64_t old = w->Vcol[j];
            if (i >= 1) vup = max2(vup, old);

            int64_t S, D, I; uint8_t code;
            int live;
            if (i == 0 && j == 0) {
                S = 0; D = NEG; I = NEG; code = 0; live = 1;
            } else {
                int64_t H = (i >= 1 && j >= 1) ? Sd + subst(p, A[i - 1], B[j - 1]) : NEG;
                int dbit = 0, ibit = 0;
                D = NEG;
                if (i >= 1) {
                    int64_t ext = Du - E, opn = Su - O - E;
                    if (ext > opn) { D = ext; dbit = 1; } else D = opn;
                }
                I = NEG;
                if (j >= 1) {
                    int64_t ext = Il - E, opn = Sl - O - E;
                    if (ext > opn) { I = ext; ibit = 1; } else I = opn;
                }
                int src = 0; int64_t m = H;          /* R4: H > D > I */
                if (D > m) { src = 1; m = D; }
                if (I > m) { src = 2; m = I; }
                int64_t thr = max2(vup, vleft) - Y;  /* R3 */
                live = m >= thr;
                if (live) S = m; else { S = NEG; D = NEG; I = NEG; }
                code = (uint8_t)(src | (dbit << 2) | (ibit << 3));
            }
            w->codes[codes_used++] = code;
            w->cS[j] = S; w->cD[j] = D; w->cI[j] = I;
            if (live) {
                w->Vcol[j] = max2(old, S);
                if (j + 1 > w->vcol_dirty) w->vcol_dirty = j + 1;
                if (first < 0) first = j;
                last = j;
                if (S > best) { best = S; bi = i; bj = j; }   /* R5: strict > in row-major order */
            }
            vleft = max2(vleft, w->Vcol[j]);
            Sl = S; Il = I; live_l = live;
        }
        int64_t hi = j - 1;
        /* current row becomes previous row */
        int64_t *t;
        t = w->pS; w->pS = w->cS; w->cS = t;
        t = w->pD; w->pD = w->cD; w->cD = t;
        plo = lo; phi = hi; pfirst = first; plast = last;
        if (first >= 0) rows = i + 1;
        else break;
    }

    out->score = best; out->i = bi; out->j = bj;
    out->explored = explored; out->rows = rows;
    out->overflow = best >= SCORE_LIMIT;

    /* traceback: from (bi, bj) in state S back to the origin */
    if (ws_ops(w, bi + bj + 1)) return -1;
    int64_t n = 0, ci = bi, cj = bj;
    int state = 0;  /* 0 S, 1 D, 2 I */
    while (ci > 0 || cj > 0) {
        uint8_t code = w->codes[w->row_off[ci] + (cj - w->row_lo[ci])];
        if (state == 0) {
            int src = code & 3;
            if (src == 0) { w->ops[n++] = 'M'; ci--; cj--; continue; }
            state = src;  /* 1 -> D, 2 -> I, same cell */
        }
        if (state == 1) { w->ops[n++] = 'D'; state = (code >> 2) & 1 ? 1 : 0; ci--; }
        else            { w->ops[n++] = 'I'; state = (code >> 3) & 1 ? 2 : 0; cj--; }
    }
    /* emitted peak -> origin; reverse to origin-outward */
    for (int64_t a = 0, b = n - 1; a < b; a++, b--) { char c = w->ops[a]; w->ops[a] = w->ops[b]; w->ops[b] = c; }
    out->nops = n;
    return 0;
}

/* ---- public entry points ------------------------------------------------------------------------- */

static int code_of(char c) {
    switch (c) {
        case 'A': case 'a': return 0;
        case 'C': case 'c': return 1;
        case 'G': case 'g': return 2;
        case 'T': case 't': return 3;
        case 'N': case 'n': return 4;  /* reading R13 */
        default: return -1;
    }
}

/* ASCII -> codes; returns index of first invalid character or -1 */
int64_t fzo_encode(const char *s, int64_t n, uint8_t *out) {
    for (int64_t k = 0; k < n; k++) {
        int c = code_of(s[k]);
        if (c < 0) return k;
        out[k] = (uint8_t)c;
    }
    return -1;
}

/* one-sided on code arrays; ops (origin-outward) copied to ops_out (capacity >= i*+j*) */
int fzo_one_sided(const uint8_t *A, int64_t M, const uint8_t *B, int64_t N, const fzo_params *p,
                  fzo_side *out, char *ops_out, int64_t ops_cap) {
    fzo_ws w; memset(&w, 0, sizeof(w));
    int rc = one_sided(A, M, B, N, p, out, &w);
    if (rc == 0) {
        if (out->nops > ops_cap) rc = -2;
        else if (out->nops) memcpy(ops_out, w.ops, (size_t)out->nops);
    }
    ws_free(&w);
    return rc;
}

typedef struct {
    const uint8_t *T, *Q, *Trev, *Qrev; int64_t tlen, qlen;
    const int64_t *seeds; int64_t n;
    const fzo_params *p;
    fzo_alignment *out;
    char **cigars;            /* per seed, malloc'd text */
    volatile int64_t next;
    volatile int err;
} job_t;

static int append_run(char **buf, int64_t *len, int64_t *cap, char op, int64_t cnt) {
    if (*len + 24 > *cap) {
        int64_t c = *cap ? *cap * 2 : 64;
        while (*len + 24 > c) c *= 2;
        char *q = (char *)realloc(*buf, (size_t)c);
        if (!q) return -1;
        *buf = q; *cap = c;
    }
    char tmp[24]; int k = 0;
    do { tmp[k++] = (char)('0' + cnt % 10); cnt /= 10; } while (cnt);
    while (k) (*buf)[(*len)++] = tmp[--k];
    (*buf)[(*len)++] = op;
    return 0;
}

/* left and right one-sided extensions of one cut point, added */
static int two_sided(job_t *J, int64_t s, fzo_ws *w, char **lops, int64_t *lops_cap) {
    const int64_t tpos = J->seeds[2 * s], qpos = J->seeds[2 * s + 1];
    fzo_alignment *a = &J->out[s];
    memset(a, 0, sizeof(*a));
    fzo_side L, Rr;
    /* left: A_k = T[tpos-k], B_k = Q[qpos-k]  ==  reversed copies starting at tlen-tpos, qlen-qpos */
    if (one_sided(J->Trev + (J->tlen - tpos), tpos, J->Qrev + (J->qlen - qpos), qpos, J->p, &L, w)) return -1;
    if (L.nops > *lops_cap) {
        char *q = (char *)realloc(*lops, (size_t)L.nops + 1);
        if (!q) return -1;
        *lops = q; *lops_cap = L.nops + 1;
    }
    if (L.nops) memcpy(*lops, w->ops, (size_t)L.nops);
    /* right: A_k = T[tpos+k-1], B_k = Q[qpos+k-1] */
    if (one_sided(J->T + tpos, J->tlen - tpos, J->Q + qpos, J->qlen - qpos, J->p, &Rr, w)) return -1;

    a->left_score = L.score; a->right_score = Rr.score; a->score = L.score + Rr.score;
    a->li = L.i; a->lj = L.j; a->ri = Rr.i; a->rj = Rr.j;
    a->t_start = tpos - L.i; a->t_end = tpos + Rr.i;
    a->q_start = qpos - L.j; a->q_end = qpos + Rr.j;
    a->l_explored = L.explored; a->r_explored = Rr.explored;
    a->flags = (a->score >= J->p->gapped_threshold ? 1 : 0)
             | ((L.i <= J->p->eager_max && L.j <= J->p->eager_max) ? 2 : 0)
             | ((Rr.i <= J->p->eager_max && Rr.j <= J->p->eager_max) ? 4 : 0)
             | ((L.overflow || Rr.overflow) ? 8 : 0);

    /* forward order: left ops are emitted origin-outward in the reversed frame, i.e. reversed here;
       right ops origin-outward are already forward.  Adjacent equal ops merge into one run (c.8). */
    char *txt = NULL; int64_t len = 0, cap = 0;
    char cur = 0; int64_t cnt = 0;
    for (int64_t k = L.nops - 1; k >= 0; k--) {
        char op = (*lops)[k];
        if (op == cur) cnt++;
        else { if (cnt && append_run(&txt, &len, &cap, cur, cnt)) return -1; cur = op; cnt = 1; }
    }
    for (int64_t k = 0; k < Rr.nops; k++) {
        char op = w->ops[k];
        if (op == cur) cnt++;
        else { if (cnt && append_run(&txt, &len, &cap, cur, cnt)) return -1; cur = op; cnt = 1; }
    }
    if (cnt && append_run(&txt, &len, &cap, cur, cnt)) return -1;
    a->cigar_len = len;
    J->cigars[s] = txt;
    return 0;
}

static void *worker(void *arg) {
    job_t *J = (job_t *)arg;
    fzo_ws w; memset(&w, 0, sizeof(w));
    char *lops = NULL; int64_t lops_cap = 0;
    for (;;) {
        int64_t s0 = __sync_fetch_and_add(&J->next, 16);
        if (s0 >= J->n || J->err) break;
        int64_t s1 = s0 + 16 < J->n ? s0 + 16 : J->n;
        for (int64_t s = s0; s < s1; s++)
            if (two_sided(J, s, &w, &lops, &lops_cap)) { J->err = 1; break; }
    }
    free(lops);
    ws_free(&w);
    return NULL;
}

/*
 * Two-sided extension of n seeds (int64 pairs tpos, qpos; 0 <= tpos <= tlen, 0 <= qpos <= qlen).
 * Results in seed order; CIGAR text concatenated into *cigar_out (malloc'd; free with fzo_free).
 * Returns 0; -1 allocation / thread failure; -2 invalid base (index in *bad); -3 seed out of range.
 */
int fzo_extend(const char *Tt, int64_t tlen, const char *Qt, int64_t qlen, const int64_t *seeds, int64_t n,
               const fzo_params *p, int nthreads, fzo_alignment *out, char **cigar_out, int64_t *cigar_bytes,
               int64_t *bad) {
    *cigar_out = NULL; *cigar_bytes = 0; *bad = -1;
    for (int64_t s = 0; s < n; s++)
        if (seeds[2 * s] < 0 || seeds[2 * s] > tlen || seeds[2 * s + 1] < 0 || seeds[2 * s + 1] > qlen) {
            *bad = s; return -3;
        }
    uint8_t *T = (uint8_t *)malloc((size_t)tlen + 1), *Q = (uint8_t *)malloc((size_t)qlen + 1);
    uint8_t *Tr = (uint8_t *)malloc((size_t)tlen + 1), *Qr = (uint8_t *)malloc((size_t)qlen + 1);
    char **cig = (char **)calloc((size_t)n + 1, sizeof(char *));
    int rc = 0;
    if (!T || !Q || !Tr || !Qr || !cig) { rc = -1; goto done; }
    int64_t b;
    if ((b = fzo_encode(Tt, tlen, T)) >= 0) { *bad = b; rc = -2; goto done; }
    if ((b = fzo_encode(Qt, qlen, Q)) >= 0) { *bad = tlen + b; rc = -2; goto done; }
    for (int64_t k = 0; k < tlen; k++) Tr[k] = T[tlen - 1 - k];
    for (int64_t k = 0; k < qlen; k++) Qr[k] = Q[qlen - 1 - k];

    job_t J;
    J.T = T; J.Q = Q; J.Trev = Tr; J.Qrev = Qr; J.tlen = tlen; J.qlen = qlen;
    J.seeds = seeds; J.n = n; J.p = p; J.out = out; J.cigars = cig; J.next = 0; J.err = 0;
    if (nthreads < 1) nthreads = 1;
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    if (!th) { rc = -1; goto done; }
    int started = 0;
    for (int k = 0; k < nthreads; k++) {
        if (pthread_create(&th[k], NULL, worker, &J)) break;
        started++;
    }
    if (!started) worker(&J);
    for (int k = 0; k < started; k++) pthread_join(th[k], NULL);
    free(th);
    if (J.err) { rc = -1; goto done; }

    int64_t total = 0;
    for (int64_t s = 0; s < n; s++) { out[s].cigar_off = total; total += out[s].cigar_len; }
    char *buf = (char *)malloc((size_t)total + 1);
    if (!buf) { rc = -1; goto done; }
    for (int64_t s = 0; s < n; s++)
        if (out[s].cigar_len) memcpy(buf + out[s].cigar_off, cig[s], (size_t)out[s].cigar_len);
    buf[total] = 0;
    *cigar_out = buf; *cigar_bytes = total;
done:
    if (cig) { for (int64_t s = 0; s < n; s++) free(cig[s]); free(cig); }
    free(T); free(Q); free(Tr); free(Qr);
    return rc;
}

void fzo_free(void *ptr) { free(ptr); }
