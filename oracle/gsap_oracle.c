/*
 * oracle/gsap_oracle.c -- TEST INFRASTRUCTURE, NOT PART OF THE PRODUCT PATH.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this library.  It shares no code, header, table or
 * helper with paper_conf_icpp_changzh24_b200/ (the CUDA path); neither side
 * includes or links the other.
 *
 * A plain, slow, obviously-correct CPU implementation of the hot path of
 * GSAP's stochastic block partitioning (Chang, Zhang & Huang, "GSAP: A
 * GPU-Accelerated Stochastic Graph Partitioner", ICPP'24).  Citations are
 * "P:<line> <section>" into /root/reference/PAPER.md; "R:<id>" refers to the
 * readings listed in DESIGN.md ("Readings of the paper"), which follow
 * SURVEY.md section 8(c).
 *
 * Deliberate differences from the CUDA path (so that the two are independent):
 *   - blockmodel rebuild: qsort of (b_src, b_dst, w) triples + run combine
 *     (CUDA: dense histogram / radix sort + RLE);
 *   - cumulative walks are linear scans (CUDA: binary search on prefix sums);
 *   - Delta S for a move / merge is computed from the *definition*: the list of
 *     blockmodel entries that change, built edge by edge from M_xy =
 *     sum_{u->w} w [b_u = x][b_w = y], then S(after) - S(before) restricted to
 *     those entries (CUDA: the decomposed o_t/i_t + 2x2-core form, and the
 *     g(a,c) intersection form for merges);
 *   - Hastings term summed edge by edge over v's adjacency (CUDA: per unique
 *     neighbour block);
 *   - merge selection is the sequential GraphChallenge loop (CUDA: parallel
 *     cycle rejection + rank prefix + pointer jumping);
 *   - entropy arithmetic in long double (x87 80-bit); decisions that floating
 *     point takes (MH accept, merge order, convergence) are taken in double,
 *     the kernel's precision.
 *
 * Parity status of each function is listed in DESIGN.md ("Oracle pins").
 *
 * Threads: single-threaded by default (the canonical run).  orc_set_threads(n)
 * lets the per-vertex / per-block loops of a batch or a merge phase (proposals,
 * Delta S, Hastings, accept) run on n OpenMP threads (SURVEY 8(d) "OpenMP
 * across the batch"): every id writes only its own outputs from the same
 * snapshot, so the results are identical for any n; everything else
 * (rebuild, sums, selection, driver) stays sequential.
 */
#include <fenv.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef long double LD;

/* ------------------------------------------------------------------------ */
/* Philox4x32-10 counter-based generator (Salmon et al., SC'11 / Random123). */
/* Replaces the paper's cuRAND lookup tables (P:168 3.2, Fig. 4); R:Z6.      */
/* ------------------------------------------------------------------------ */
void orc_philox(const uint32_t *ctr, const uint32_t *key, uint32_t *out)
{
    uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
    uint32_t k0 = key[0], k1 = key[1];
    int round;
    for (round = 0; round < 10; ++round) {
        uint64_t p0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
        uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
        uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
        uint32_t n0 = hi1 ^ c1 ^ k0;
        uint32_t n1 = lo1;
        uint32_t n2 = hi0 ^ c3 ^ k1;
        uint32_t n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* the random words for (id, draw j, iteration, outer round, phase); R:O.3 */
static void draws(uint64_t seed, uint32_t id, uint32_t j, uint32_t itr,
                  uint32_t outer, uint32_t phase, uint32_t w[4])
{
    uint32_t ctr[4], key[2];
    ctr[0] = id; ctr[1] = j; ctr[2] = itr; ctr[3] = (outer << 1) | phase;
    key[0] = (uint32_t)(seed & 0xffffffffu);
    key[1] = (uint32_t)(seed >> 32);
    orc_philox(ctr, key, w);
}

/* floor(w * T / 2^32): an integer uniformly-ish drawn from [0, T) */
static uint64_t pick(uint32_t w, uint64_t T)
{
    return ((uint64_t)w * T) >> 32;
}

/* ------------------------------------------------------------------------ */
/* Graph: out lists in the caller's CSR order, in lists ordered by source id */
/* (then CSR position).  P:257 3.4 ("Graph_adjPtr / adjNbr / adjWgt").       */
/* ------------------------------------------------------------------------ */
typedef struct {
    int32_t V;
    int64_t E;    /* number of edge entries */
    int64_t W;    /* total edge weight (the "E" of Eq. 2; R:Z22) */
    int64_t *optr; int32_t *odst; int64_t *ow;
    int64_t *iptr; int32_t *isrc; int64_t *iw;
    int64_t *kout, *kin;   /* weighted out / in degree (self-loop in both) */
} OG;

/* ------------------------------------------------------------------------ */
/* Blockmodel: M_xy = total weight of edges u->w with b_u = x, b_w = y       */
/* (P:56 2.1; R:Z1).  CSR (rows ascending column) + CSC (columns ascending   */
/* row) as in P:152-159 3.1 ("six arrays"), out/in block degrees.    */
/* ------------------------------------------------------------------------ */
typedef struct {
    int32_t B;
    int64_t nnz;
    int64_t *rptr; int32_t *rcol; int64_t *rcnt;
    int64_t *cptr; int32_t *crow; int64_t *ccnt;
    int64_t *dout, *din;
} OBM;

typedef struct {
    OG g;
    int32_t *b;
    int32_t B;
    OBM bm;
    int table_mode;     /* N4 ablation: 1 = the paper-literal shared lookup table */
    int32_t *mt;        /* mt[x]: one weighted neighbour block of block x, or -1 */
} OState;

static void *xmalloc(size_t n)
{
    void *p = malloc(n ? n : 1);
    if (!p) abort();
    return p;
}
static void *xcalloc(size_t n, size_t s)
{
    void *p = calloc(n ? n : 1, s ? s : 1);
    if (!p) abort();
    return p;
}

static void bm_free(OBM *m)
{
    free(m->rptr); free(m->rcol); free(m->rcnt);
    free(m->cptr); free(m->crow); free(m->ccnt);
    free(m->dout); free(m->din);
    memset(m, 0, sizeof(*m));
}

typedef struct { int32_t x, y; int64_t w; } Trip;

static int cmp_trip(const void *a, const void *b)
{
    const Trip *p = (const Trip *)a, *q = (const Trip *)b;
    if (p->x != q->x) return p->x < q->x ? -1 : 1;
    if (p->y != q->y) return p->y < q->y ? -1 : 1;
    return 0;
}

/* Alg. 2 (P:268-283 3.4), as its definition: the blockmodel of partition b. */
static void rebuild(OState *st)
{
    const OG *g = &st->g;
    OBM *m = &st->bm;
    int32_t B = st->B, u, x;
    int64_t e, n = 0, k, i;
    Trip *t = (Trip *)xmalloc(sizeof(Trip) * (size_t)(g->E ? g->E : 1));
    bm_free(m);
    m->B = B;
    for (u = 0; u < g->V; ++u)
        for (e = g->optr[u]; e < g->optr[u + 1]; ++e) {
            t[n].x = st->b[u];
            t[n].y = st->b[g->odst[e]];
            t[n].w = g->ow[e];
            ++n;
        }
    qsort(t, (size_t)n, sizeof(Trip), cmp_trip);
    /* combine runs of equal (x, y) */
    k = 0;
    for (i = 0; i < n; ++i) {
        if (k > 0 && t[k - 1].x == t[i].x && t[k - 1].y == t[i].y)
            t[k - 1].w += t[i].w;
        else
            t[k++] = t[i];
    }
    m->nnz = k;
    m->rptr = (int64_t *)xcalloc((size_t)B + 1, sizeof(int64_t));
    m->rcol = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)(k ? k : 1));
    m->rcnt = (int64_t *)xmalloc(sizeof(int64_t) * (size_t)(k ? k : 1));
    m->dout = (int64_t *)xcalloc((size_t)B, sizeof(int64_t));
    m->din = (int64_t *)xcalloc((size_t)B, sizeof(int64_t));
    for (i = 0; i < k; ++i) {
        m->rptr[t[i].x + 1]++;
        m->rcol[i] = t[i].y;
        m->rcnt[i] = t[i].w;
        m->dout[t[i].x] += t[i].w;
        m->din[t[i].y] += t[i].w;
    }
    for (x = 0; x < B; ++x) m->rptr[x + 1] += m->rptr[x];
    /* CSC: the same entries keyed (y, x) */
    for (i = 0; i < k; ++i) {
        int32_t tmp = t[i].x;
        t[i].x = t[i].y;
        t[i].y = tmp;
    }
    qsort(t, (size_t)k, sizeof(Trip), cmp_trip);
    m->cptr = (int64_t *)xcalloc((size_t)B + 1, sizeof(int64_t));
    m->crow = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)(k ? k : 1));
    m->ccnt = (int64_t *)xmalloc(sizeof(int64_t) * (size_t)(k ? k : 1));
    for (i = 0; i < k; ++i) {
        m->cptr[t[i].x + 1]++;
        m->crow[i] = t[i].y;
        m->ccnt[i] = t[i].w;
    }
    for (x = 0; x < B; ++x) m->cptr[x + 1] += m->cptr[x];
    free(t);
}

/* M_xy by binary search in CSR row x (0 if absent) */
static int64_t M_at(const OBM *m, int32_t x, int32_t y)
{
    int64_t lo = m->rptr[x], hi = m->rptr[x + 1];
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (m->rcol[mid] < y) lo = mid + 1;
        else hi = mid;
    }
    if (lo < m->rptr[x + 1] && m->rcol[lo] == y) return m->rcnt[lo];
    return 0;
}

static int64_t deg(const OBM *m, int32_t x) { return m->dout[x] + m->din[x]; }

/* f(m) = m ln m, f(0) = 0 */
static LD fl(LD m) { return m > 0 ? m * logl(m) : 0.0L; }

/* ------------------------------------------------------------------------ */
/* Description length, Eq. 1-2 (P:56-65 2.1), readings Z1-Z4, Z22:          */
/*   S   = -sum_xy M_xy ln(M_xy / (dout_x din_y))                            */
/*       = -sum f(M_xy) + sum f(dout_x) + sum f(din_y)                       */
/*   MDL = E h(B^2/E) + V ln B + S,  h(x) = (1+x) ln(1+x) - x ln x           */
/* model_term = 1 selects the GraphChallenge-code variant (R:Z3).           */
/* ------------------------------------------------------------------------ */
static LD data_term(const OBM *m)
{
    LD s = 0.0L;
    int64_t i;
    int32_t x;
    for (i = 0; i < m->nnz; ++i) s -= fl((LD)m->rcnt[i]);
    for (x = 0; x < m->B; ++x) s += fl((LD)m->dout[x]) + fl((LD)m->din[x]);
    return s;
}

static LD model_term(int64_t W, int32_t V, int32_t B, int variant)
{
    LD E = (LD)W, x, t;
    if (W <= 0) return (LD)V * logl((LD)B);
    x = (LD)B * (LD)B / E;
    if (variant == 1)
        t = E * (1.0L + x) * logl(1.0L + x) - x * logl(x);
    else
        t = E * ((1.0L + x) * logl(1.0L + x) - x * logl(x));
    return t + (LD)V * logl((LD)B);
}

double orc_mdl_of(OState *st, int variant, double *data_out)
{
    LD d = data_term(&st->bm);
    if (data_out) *data_out = (double)d;
    return (double)(model_term(st->g.W, st->g.V, st->B, variant) + d);
}

/* ------------------------------------------------------------------------ */
/* Proposals, Alg. 1 (P:180-201 3.2) with the P:166 description; readings   */
/* Z6-Z9 (O.4 in SURVEY.md 8c).  Linear cumulative walks.                   */
/* ------------------------------------------------------------------------ */

/* the weighted neighbour of block u at offset p of (out-row u ++ in-col u),
 * skipping id `skip` in both (skip < 0: skip nothing) */
static int32_t walk_block(const OBM *m, int32_t u, uint64_t p, int32_t skip)
{
    uint64_t acc = 0;
    int64_t i;
    for (i = m->rptr[u]; i < m->rptr[u + 1]; ++i) {
        if (m->rcol[i] == skip) continue;
        acc += (uint64_t)m->rcnt[i];
        if (p < acc) return m->rcol[i];
    }
    for (i = m->cptr[u]; i < m->cptr[u + 1]; ++i) {
        if (m->crow[i] == skip) continue;
        acc += (uint64_t)m->ccnt[i];
        if (p < acc) return m->crow[i];
    }
    return -1; /* unreachable when p < total */
}

/* ------------------------------------------------------------------------ */
/* N4 ablation: the paper's lookup tables (P:168 3.2, Fig. 4; Alg. 1 lines   */
/* 5 and 10): one multinomial draw of a neighbour block per block, */
/* shared by every proposal of the merge phase / MOVE batch.  The draw for   */
/* block x uses its own Philox counter (x, TABLE_J | key, itr, outer<<1|ph). */
/* ------------------------------------------------------------------------ */
#define ORC_TABLE_J 0x40000000u

static void build_table(OState *st, uint64_t seed, uint32_t j, uint32_t itr, uint32_t outer, uint32_t phase)
{
    int32_t x;
    uint32_t w[4];
    if (!st->mt) st->mt = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)(st->g.V ? st->g.V : 1));
    for (x = 0; x < st->B; ++x) {
        uint64_t d = (uint64_t)deg(&st->bm, x);
        draws(seed, (uint32_t)x, j, itr, outer, phase, w);
        st->mt[x] = d ? walk_block(&st->bm, x, pick(w[0], d), -1) : -1;
    }
}

static int32_t propose_move(const OState *st, uint64_t seed, uint32_t outer,
                            uint32_t itr, int32_t v)
{
    const OG *g = &st->g;
    const OBM *m = &st->bm;
    uint32_t w[4];
    uint64_t K = (uint64_t)(g->kout[v] + g->kin[v]), p, acc = 0, B = (uint64_t)st->B;
    int32_t n = -1, u;
    uint64_t du;
    int64_t e;
    draws(seed, (uint32_t)v, 0, itr, outer, 1u, w);
    if (K == 0) return (int32_t)pick(w[2], B);            /* P:166, R:Z8 */
    p = pick(w[0], K);
    for (e = g->optr[v]; e < g->optr[v + 1] && n < 0; ++e) {
        acc += (uint64_t)g->ow[e];
        if (p < acc) n = g->odst[e];
    }
    for (e = g->iptr[v]; e < g->iptr[v + 1] && n < 0; ++e) {
        acc += (uint64_t)g->iw[e];
        if (p < acc) n = g->isrc[e];
    }
    u = st->b[n];
    du = (uint64_t)deg(m, u);
    /* x <= B/(B+deg u) -> random block, as an exact integer test (R:Z9) */
    if ((uint64_t)w[1] * (B + du) <= (B << 32)) return (int32_t)pick(w[2], B);
    if (st->table_mode) return st->mt[u];      /* N4: Alg. 1 line 10 */
    return walk_block(m, u, pick(w[2], du), -1);
}

static int32_t propose_merge(const OState *st, uint64_t seed, uint32_t outer,
                             int32_t r, uint32_t j)
{
    const OBM *m = &st->bm;
    uint32_t w[4];
    uint64_t B = (uint64_t)st->B, K = (uint64_t)deg(m, r), du, T;
    int32_t u, s;
    draws(seed, (uint32_t)r, j, 0u, outer, 0u, w);
    if (K == 0) goto random;
    if (st->table_mode) {                      /* N4: Alg. 1 lines 5-10 with the shared table */
        u = st->mt[r];
        du = (uint64_t)deg(m, u);
        if ((uint64_t)w[1] * (B + du) <= (B << 32)) goto random;
        s = st->mt[u];
        if (s >= 0 && s != r) return s;
        goto random;                           /* an outcome equal to r is redrawn (reading N4) */
    }
    u = walk_block(m, r, pick(w[0], K), -1);
    du = (uint64_t)deg(m, u);
    if ((uint64_t)w[1] * (B + du) <= (B << 32)) goto random;
    T = du - (uint64_t)M_at(m, u, r) - (uint64_t)M_at(m, r, u);
    if (T == 0) goto random;
    return walk_block(m, u, pick(w[2], T), r);   /* merges exclude r (R:Z6) */
random:
    s = (int32_t)pick(w[2], B - 1);
    if (s >= r) s += 1;
    return s;
}

/* ------------------------------------------------------------------------ */
/* Changed-entry lists ("delta lists"), built straight from the definition  */
/* of M: every edge that changes block endpoints subtracts its weight from  */
/* its old (b_src, b_dst) entry and adds it to its new one.                 */
/* ------------------------------------------------------------------------ */
typedef struct { Trip *t; int64_t n, cap; } DL;

static void dl_push(DL *d, int32_t x, int32_t y, int64_t w)
{
    if (d->n == d->cap) {
        d->cap = d->cap ? 2 * d->cap : 64;
        d->t = (Trip *)realloc(d->t, sizeof(Trip) * (size_t)d->cap);
        if (!d->t) abort();
    }
    d->t[d->n].x = x; d->t[d->n].y = y; d->t[d->n].w = w;
    d->n++;
}

static void dl_combine(DL *d)
{
    int64_t i, k = 0;
    qsort(d->t, (size_t)d->n, sizeof(Trip), cmp_trip);
    for (i = 0; i < d->n; ++i) {
        if (k > 0 && d->t[k - 1].x == d->t[i].x && d->t[k - 1].y == d->t[i].y)
            d->t[k - 1].w += d->t[i].w;
        else
            d->t[k++] = d->t[i];
    }
    d->n = k;
}

static int64_t dl_at(const DL *d, int32_t x, int32_t y)
{
    int64_t lo = 0, hi = d->n;
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        const Trip *t = &d->t[mid];
        if (t->x < x || (t->x == x && t->y < y)) lo = mid + 1;
        else hi = mid;
    }
    if (lo < d->n && d->t[lo].x == x && d->t[lo].y == y) return d->t[lo].w;
    return 0;
}

/* the changed entries of M when vertex v moves r -> s (Eq. 7) */
static void move_deltas(const OState *st, int32_t v, int32_t s, DL *d)
{
    const OG *g = &st->g;
    int32_t r = st->b[v];
    int64_t e;
    d->n = 0;
    for (e = g->optr[v]; e < g->optr[v + 1]; ++e) {
        int32_t w = g->odst[e];
        int32_t y_old = st->b[w], y_new = (w == v) ? s : st->b[w];
        dl_push(d, r, y_old, -g->ow[e]);
        dl_push(d, s, y_new, +g->ow[e]);
    }
    for (e = g->iptr[v]; e < g->iptr[v + 1]; ++e) {
        int32_t w = g->isrc[e];
        if (w == v) continue;          /* the self-loop was handled as an out-edge */
        dl_push(d, st->b[w], r, -g->iw[e]);
        dl_push(d, st->b[w], s, +g->iw[e]);
    }
    dl_combine(d);
}

/* S(after) - S(before) over the changed entries and the changed degrees */
static LD dS_of_deltas(const OBM *m, const DL *d, int32_t r, int32_t s,
                       int64_t dout_shift, int64_t din_shift)
{
    LD dS = 0.0L;
    int64_t i;
    for (i = 0; i < d->n; ++i) {
        int64_t before, after;
        if (d->t[i].w == 0) continue;
        before = M_at(m, d->t[i].x, d->t[i].y);
        after = before + d->t[i].w;
        dS -= fl((LD)after) - fl((LD)before);
    }
    /* degrees: out(r) -= shift, out(s) += shift, same for in */
    dS += fl((LD)(m->dout[r] - dout_shift)) - fl((LD)m->dout[r]);
    dS += fl((LD)(m->dout[s] + dout_shift)) - fl((LD)m->dout[s]);
    dS += fl((LD)(m->din[r] - din_shift)) - fl((LD)m->din[r]);
    dS += fl((LD)(m->din[s] + din_shift)) - fl((LD)m->din[s]);
    return dS;
}

/*
 * Vertex move v: r -> s.  Delta S (Eq. 7), the Hastings correction and the
 * Metropolis-Hastings acceptance (P:34, P:67 2.1, P:141 3; R:Z5, Z13, Z15,
 * Z26): H = p_bwd / p_fwd with
 *   p_fwd = sum over v's adjacency entries (out list ++ in list, a self-loop
 *           in both) of  w * (M_ts + M_st + 1) / (d_t + B),  t = b[nbr],
 *   p_bwd = the same over the after-state, toward r, with the after-state
 *           block of each neighbour (v itself is in s after the move),
 * accept iff u <= min(1, exp(-beta dS) H), u = (w3 + 1/2) 2^-32.
 */
static void eval_move(const OState *st, DL *d, uint64_t seed, uint32_t outer,
                      uint32_t itr, double beta, int32_t v, int32_t s,
                      double *dS_out, double *H_out, double *p_out, uint8_t *acc_out)
{
    const OG *g = &st->g;
    const OBM *m = &st->bm;
    int32_t r = st->b[v], B = st->B;
    uint32_t w[4];
    LD dS, pf = 0.0L, pb = 0.0L, H;
    double p, u;
    int64_t e, kout = g->kout[v], kin = g->kin[v];
    draws(seed, (uint32_t)v, 0, itr, outer, 1u, w);
    if (s == r) {                      /* R:Z13: no move */
        *dS_out = 0.0; *H_out = 1.0; *p_out = 0.0; *acc_out = 0;
        return;
    }
    move_deltas(st, v, s, d);
    dS = dS_of_deltas(m, d, r, s, kout, kin);
    /* Hastings, edge by edge over the proposal law's support */
    for (int pass = 0; pass < 2; ++pass) {
        int64_t lo = pass ? g->iptr[v] : g->optr[v];
        int64_t hi = pass ? g->iptr[v + 1] : g->optr[v + 1];
        for (e = lo; e < hi; ++e) {
            int32_t nb = pass ? g->isrc[e] : g->odst[e];
            LD wt = (LD)(pass ? g->iw[e] : g->ow[e]);
            int32_t t = st->b[nb];                 /* before the move */
            int32_t t2 = (nb == v) ? s : st->b[nb]; /* after the move */
            LD dt = (LD)deg(m, t);
            LD dt2 = (LD)deg(m, t2) + (t2 == r ? -(LD)(kout + kin) : 0.0L)
                                    + (t2 == s ? (LD)(kout + kin) : 0.0L);
            LD a = (LD)(M_at(m, t, s) + M_at(m, s, t)) + 1.0L;
            LD a2 = (LD)(M_at(m, t2, r) + dl_at(d, t2, r) +
                         M_at(m, r, t2) + dl_at(d, r, t2)) + 1.0L;
            pf += wt * a / (dt + (LD)B);
            pb += wt * a2 / (dt2 + (LD)B);
        }
    }
    H = (kout + kin == 0) ? 1.0L : pb / pf;
    p = exp(-beta * (double)dS) * (double)H;
    u = ((double)w[3] + 0.5) * (1.0 / 4294967296.0);
    *dS_out = (double)dS;
    *H_out = (double)H;
    *p_out = p;
    *acc_out = (uint8_t)(u <= p);
}

/* Block merge r into s: Eq. 4-6 (P:211-232 3.3) in exact form (R:Z11, Z12). */
static double eval_merge(const OState *st, DL *d, int32_t r, int32_t s)
{
    const OBM *m = &st->bm;
    int64_t i;
    LD dS;
    d->n = 0;
    for (i = m->rptr[r]; i < m->rptr[r + 1]; ++i) {
        int32_t y = m->rcol[i];
        dl_push(d, r, y, -m->rcnt[i]);
        dl_push(d, s, (y == r) ? s : y, +m->rcnt[i]);
    }
    for (i = m->cptr[r]; i < m->cptr[r + 1]; ++i) {
        int32_t x = m->crow[i];
        if (x == r) continue;          /* (r, r) was moved with row r */
        dl_push(d, x, r, -m->ccnt[i]);
        dl_push(d, x, s, +m->ccnt[i]);
    }
    dl_combine(d);
    dS = 0.0L;
    for (i = 0; i < d->n; ++i) {
        int64_t before, after;
        if (d->t[i].w == 0) continue;
        before = M_at(m, d->t[i].x, d->t[i].y);
        after = before + d->t[i].w;
        dS -= fl((LD)after) - fl((LD)before);
    }
    dS += fl((LD)(m->dout[s] + m->dout[r])) - fl((LD)m->dout[s]) - fl((LD)m->dout[r]);
    dS += fl((LD)(m->din[s] + m->din[r])) - fl((LD)m->din[s]) - fl((LD)m->din[r]);
    return (double)dS;
}

/* ------------------------------------------------------------------------ */
/* Perform-merge (P:141 3, P:232 3.3): blocks in ascending (dS_best, id)     */
/* order; the sequential GraphChallenge loop; relabel to the ranks of the   */
/* labels present in b (R:Z16-Z18).                                          */
/* ------------------------------------------------------------------------ */
typedef struct { double key; int32_t id; } KeyId;

static int cmp_keyid(const void *a, const void *b)
{
    const KeyId *p = (const KeyId *)a, *q = (const KeyId *)b;
    if (p->key < q->key) return -1;
    if (p->key > q->key) return 1;
    return p->id < q->id ? -1 : (p->id > q->id ? 1 : 0);
}

static int32_t select_merges(OState *st, const int32_t *best, const double *dS,
                             int32_t K, int32_t *label_out)
{
    int32_t B = st->B, i, x, num = 0, newB = 0, v;
    KeyId *ord = (KeyId *)xmalloc(sizeof(KeyId) * (size_t)B);
    int32_t *map = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)B);
    int32_t *rank = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)B);
    uint8_t *present = (uint8_t *)xcalloc((size_t)B, 1);
    for (i = 0; i < B; ++i) {
        ord[i].key = (dS[i] == 0.0) ? 0.0 : dS[i];   /* -0.0 -> +0.0 */
        ord[i].id = i;
        map[i] = i;
    }
    qsort(ord, (size_t)B, sizeof(KeyId), cmp_keyid);
    for (i = 0; i < B && num < K; ++i) {
        int32_t from = ord[i].id, to = map[best[from]];
        if (to != from) {
            for (x = 0; x < B; ++x)
                if (map[x] == from) map[x] = to;
            ++num;
        }
    }
    for (v = 0; v < st->g.V; ++v) present[map[st->b[v]]] = 1;
    for (x = 0; x < B; ++x) rank[x] = present[x] ? newB++ : -1;
    for (v = 0; v < st->g.V; ++v) st->b[v] = rank[map[st->b[v]]];
    if (label_out)
        for (x = 0; x < B; ++x) label_out[x] = rank[map[x]];
    st->B = newB;
    free(ord); free(map); free(rank); free(present);
    rebuild(st);
    return newB;
}

/* ------------------------------------------------------------------------ */
/* Public (ctypes) interface, mirroring the C-ABI of the CUDA library with  */
/* an orc_ prefix.                                                           */
/* ------------------------------------------------------------------------ */
void *orc_create(int32_t V, const int64_t *rowptr, const int32_t *col, const int32_t *wgt)
{
    OState *st;
    OG *g;
    int64_t E, e, *fill;
    if (V < 0) return NULL;
    E = rowptr[V];
    st = (OState *)xcalloc(1, sizeof(OState));
    g = &st->g;
    int32_t u;
    g->V = V; g->E = E; g->W = 0;
    g->optr = (int64_t *)xmalloc(sizeof(int64_t) * ((size_t)V + 1));
    g->odst = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)(E ? E : 1));
    g->ow = (int64_t *)xmalloc(sizeof(int64_t) * (size_t)(E ? E : 1));
    g->iptr = (int64_t *)xcalloc((size_t)V + 1, sizeof(int64_t));
    g->isrc = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)(E ? E : 1));
    g->iw = (int64_t *)xmalloc(sizeof(int64_t) * (size_t)(E ? E : 1));
    g->kout = (int64_t *)xcalloc((size_t)V, sizeof(int64_t));
    g->kin = (int64_t *)xcalloc((size_t)V, sizeof(int64_t));
    memcpy(g->optr, rowptr, sizeof(int64_t) * ((size_t)V + 1));
    for (e = 0; e < E; ++e) {
        g->odst[e] = col[e];
        g->ow[e] = wgt ? wgt[e] : 1;
        g->W += g->ow[e];
        g->iptr[col[e] + 1]++;
    }
    for (u = 0; u < V; ++u) g->iptr[u + 1] += g->iptr[u];
    fill = (int64_t *)xcalloc((size_t)V, sizeof(int64_t));
    for (u = 0; u < V; ++u)
        for (e = g->optr[u]; e < g->optr[u + 1]; ++e) {
            int32_t w = g->odst[e];
            int64_t pos = g->iptr[w] + fill[w]++;
            g->isrc[pos] = u;
            g->iw[pos] = g->ow[e];
            g->kout[u] += g->ow[e];
            g->kin[w] += g->ow[e];
        }
    free(fill);
    st->b = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)(V ? V : 1));
    for (u = 0; u < V; ++u) st->b[u] = u;
    st->B = V;
    rebuild(st);
    return st;
}

void orc_destroy(void *h)
{
    OState *st = (OState *)h;
    if (!st) return;
    free(st->g.optr); free(st->g.odst); free(st->g.ow);
    free(st->g.iptr); free(st->g.isrc); free(st->g.iw);
    free(st->g.kout); free(st->g.kin);
    free(st->b);
    free(st->mt);
    bm_free(&st->bm);
    free(st);
}

/* N4 ablation switch: 0 = fresh draws (R:Z6, default), 1 = shared table */
void orc_set_proposal_mode(void *h, int mode)
{
    ((OState *)h)->table_mode = mode == 1;
}

/* the shared table as the next proposal call would build it (pins) */
void orc_table(void *h, uint64_t seed, uint32_t j, uint32_t itr, uint32_t outer, uint32_t phase, int32_t *out)
{
    OState *st = (OState *)h;
    build_table(st, seed, j, itr, outer, phase);
    memcpy(out, st->mt, sizeof(int32_t) * (size_t)st->B);
}

void orc_set_partition(void *h, const int32_t *b, int32_t B)
{
    OState *st = (OState *)h;
    memcpy(st->b, b, sizeof(int32_t) * (size_t)st->g.V);
    st->B = B;
    rebuild(st);
}

void orc_set_b_norebuild(void *h, const int32_t *b, int32_t B)
{
    OState *st = (OState *)h;
    memcpy(st->b, b, sizeof(int32_t) * (size_t)st->g.V);
    st->B = B;
}

int32_t orc_get_partition(void *h, int32_t *b)
{
    OState *st = (OState *)h;
    if (b) memcpy(b, st->b, sizeof(int32_t) * (size_t)st->g.V);
    return st->B;
}

void orc_rebuild(void *h) { rebuild((OState *)h); }

int64_t orc_nnz(void *h) { return ((OState *)h)->bm.nnz; }

int64_t orc_total_weight(void *h) { return ((OState *)h)->g.W; }

/* cum arrays are the inclusive prefix of cnt within each row / column */
void orc_get_blockmodel(void *h, int64_t *rptr, int32_t *rcol, int64_t *rcnt, int64_t *rcum,
                        int64_t *cptr, int32_t *crow, int64_t *ccnt, int64_t *ccum,
                        int64_t *dout, int64_t *din)
{
    OState *st = (OState *)h;
    OBM *m = &st->bm;
    int32_t x;
    int64_t i, B = m->B;
    if (rptr) memcpy(rptr, m->rptr, sizeof(int64_t) * (size_t)(B + 1));
    if (rcol) memcpy(rcol, m->rcol, sizeof(int32_t) * (size_t)m->nnz);
    if (rcnt) memcpy(rcnt, m->rcnt, sizeof(int64_t) * (size_t)m->nnz);
    if (cptr) memcpy(cptr, m->cptr, sizeof(int64_t) * (size_t)(B + 1));
    if (crow) memcpy(crow, m->crow, sizeof(int32_t) * (size_t)m->nnz);
    if (ccnt) memcpy(ccnt, m->ccnt, sizeof(int64_t) * (size_t)m->nnz);
    if (dout) memcpy(dout, m->dout, sizeof(int64_t) * (size_t)B);
    if (din) memcpy(din, m->din, sizeof(int64_t) * (size_t)B);
    for (x = 0; x < m->B; ++x) {
        int64_t a = 0, c = 0;
        for (i = m->rptr[x]; i < m->rptr[x + 1]; ++i) {
            a += m->rcnt[i];
            if (rcum) rcum[i] = a;
        }
        for (i = m->cptr[x]; i < m->cptr[x + 1]; ++i) {
            c += m->ccnt[i];
            if (ccum) ccum[i] = c;
        }
    }
}

double orc_mdl(void *h, int variant, double *data_out)
{
    return orc_mdl_of((OState *)h, variant, data_out);
}

static int g_threads = 1;

/* OpenMP threads of the per-id loops (1 = the canonical single-threaded run);
 * returns the number in effect (1 if built without OpenMP) */
int32_t orc_set_threads(int32_t n)
{
#ifdef _OPENMP
    g_threads = n < 1 ? 1 : n;
#else
    (void)n;
    g_threads = 1;
#endif
    return g_threads;
}

/* phase 0 = MERGE (ids are blocks, P draws each), 1 = MOVE (ids are vertices) */
void orc_propose(void *h, int phase, uint64_t seed, uint32_t outer, uint32_t itr,
                 int32_t first, int32_t count, int32_t P, int32_t *s_out)
{
    OState *st = (OState *)h;
    int32_t i, j;
    if (st->table_mode)   /* N4: the shared table of this MOVE batch (keyed by first) / merge phase */
        build_table(st, seed, phase == 1 ? (ORC_TABLE_J | ((uint32_t)first & 0x3fffffffu)) : ORC_TABLE_J,
                    phase == 1 ? itr : 0u, outer, (uint32_t)phase);
#pragma omp parallel for private(j) schedule(dynamic, 256) num_threads(g_threads) if (g_threads > 1)
    for (i = 0; i < count; ++i) {
        if (phase == 1)
            s_out[i] = propose_move(st, seed, outer, itr, first + i);
        else
            for (j = 0; j < P; ++j)
                s_out[(int64_t)i * P + j] = propose_merge(st, seed, outer, first + i, (uint32_t)j);
    }
}

void orc_delta_move(void *h, uint64_t seed, uint32_t outer, uint32_t itr, double beta,
                    int32_t first, int32_t count, const int32_t *s,
                    double *dS, double *H, double *p, uint8_t *acc)
{
    OState *st = (OState *)h;
#pragma omp parallel num_threads(g_threads) if (g_threads > 1)
    {
        DL d = {0, 0, 0};   /* scratch per thread */
        int32_t i;
#pragma omp for schedule(dynamic, 256)
        for (i = 0; i < count; ++i)
            eval_move(st, &d, seed, outer, itr, beta, first + i, s[i], &dS[i], &H[i], &p[i], &acc[i]);
        free(d.t);
    }
}

void orc_delta_merge(void *h, int32_t first, int32_t count, int32_t P,
                     const int32_t *s, double *dS)
{
    OState *st = (OState *)h;
    int64_t n = (int64_t)count * P;
#pragma omp parallel num_threads(g_threads) if (g_threads > 1)
    {
        DL d = {0, 0, 0};   /* scratch per thread */
        int64_t i;
#pragma omp for schedule(dynamic, 256)
        for (i = 0; i < n; ++i)
            dS[i] = eval_merge(st, &d, first + (int32_t)(i / P), s[i]);
        free(d.t);
    }
}

/* best proposal per block: argmin_j with strict <, first j wins (R:Z16) */
void orc_best_merges(int32_t count, int32_t P, const int32_t *s, const double *dS,
                     int32_t *best, double *dSbest)
{
    int32_t i, j;
    for (i = 0; i < count; ++i) {
        int64_t o = (int64_t)i * P;
        int32_t bj = 0;
        for (j = 1; j < P; ++j)
            if (dS[o + j] < dS[o + bj]) bj = j;
        best[i] = s[o + bj];
        dSbest[i] = dS[o + bj];
    }
}

int32_t orc_select_merges(void *h, const int32_t *best, const double *dS, int32_t K,
                          int32_t *label_out)
{
    return select_merges((OState *)h, best, dS, K, label_out);
}

/* apply accepted moves of vertices [first, first+count) (no rebuild) */
void orc_apply_moves(void *h, int32_t first, int32_t count, const int32_t *s, const uint8_t *acc)
{
    OState *st = (OState *)h;
    int32_t i;
    for (i = 0; i < count; ++i)
        if (acc[i]) st->b[first + i] = s[i];
}

/* ------------------------------------------------------------------------ */
/* Phases and the golden-section driver (P:34 1, P:61-67 2.1, P:137-141 3,  */
/* Table 2; readings Z10, Z17-Z21).             */
/* ------------------------------------------------------------------------ */
typedef struct {
    uint64_t seed;
    double beta;
    double reduction_rate;
    int32_t num_proposals;
    int32_t max_nodal_itr;
    double thresh1, thresh2;
    int32_t window;
    int32_t num_batches;
    int32_t model_term;
    int32_t max_rounds;
} OParams;

typedef struct {
    int64_t n_move_prop, n_move_acc, n_merge_prop;
    int32_t rounds, mcmc_itr_total;
} OStats;

/* one merge phase: every block proposes P merges; K of them are carried out */
static void merge_phase(OState *st, const OParams *pr, uint32_t outer, int32_t K, OStats *stats)
{
    int32_t B = st->B, P = pr->num_proposals;
    int32_t *s = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)B * (size_t)P);
    double *dS = (double *)xmalloc(sizeof(double) * (size_t)B * (size_t)P);
    int32_t *best = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)B);
    double *dSb = (double *)xmalloc(sizeof(double) * (size_t)B);
    orc_propose(st, 0, pr->seed, outer, 0, 0, B, P, s);
    orc_delta_merge(st, 0, B, P, s, dS);
    orc_best_merges(B, P, s, dS, best, dSb);
    select_merges(st, best, dSb, K, NULL);
    if (stats) stats->n_merge_prop += (int64_t)B * P;
    free(s); free(dS); free(best); free(dSb);
}

/* one MCMC batch [first, first+count): snapshot reads, then apply, rebuild */
static double mcmc_batch(OState *st, const OParams *pr, uint32_t outer, uint32_t itr,
                         int32_t first, int32_t count, OStats *stats)
{
    int32_t *s = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)(count ? count : 1));
    double *dS = (double *)xmalloc(sizeof(double) * (size_t)(count ? count : 1));
    double *H = (double *)xmalloc(sizeof(double) * (size_t)(count ? count : 1));
    double *p = (double *)xmalloc(sizeof(double) * (size_t)(count ? count : 1));
    uint8_t *acc = (uint8_t *)xmalloc((size_t)(count ? count : 1));
    double D = 0.0;
    int32_t i;
    orc_propose(st, 1, pr->seed, outer, itr, first, count, 1, s);
    orc_delta_move(st, pr->seed, outer, itr, pr->beta, first, count, s, dS, H, p, acc);
    for (i = 0; i < count; ++i)
        if (acc[i]) {
            D += dS[i];
            if (stats) stats->n_move_acc++;
        }
    orc_apply_moves(st, first, count, s, acc);
    rebuild(st);
    if (stats) stats->n_move_prop += count;
    free(s); free(dS); free(H); free(p); free(acc);
    return D;
}

/* The convergence test after MCMC iteration itr (P:141 3; Table 2
 * "delta_entropy_threshold", "delta_entropy_moving_avg_window"; R:Z19, Z20):
 * GraphChallenge's slice D[itr-w+1 : itr) -- for the default w = 3 the two
 * iterations BEFORE itr, not itr itself -- and the MDL of the state AFTER
 * iteration itr:  stop iff  -mean(slice) < thresh * MDL.  No test before
 * itr = w - 1; an empty slice (w = 1) has mean 0. */
static int mcmc_converged(const double *Dh, int32_t itr, int32_t window, double thresh, double mdl)
{
    double sum = 0.0, mean;
    int32_t j, n = 0;
    if (itr < window - 1) return 0;
    for (j = itr - window + 1; j < itr; ++j) { sum += Dh[j]; ++n; }
    mean = n ? sum / n : 0.0;
    return -mean < thresh * mdl;
}

/* MCMC phase; returns the number of iterations run.  D_out (nullable,
 * max_nodal_itr entries): D[itr] = sum of the accepted (stale) dS of
 * iteration itr, batches in order (R:Z20). */
static int32_t mcmc_phase(OState *st, const OParams *pr, uint32_t outer, double thresh, OStats *stats,
                          double *D_out)
{
    int32_t V = st->g.V, nb = pr->num_batches, itr, k;
    int32_t bs = (V + nb - 1) / nb;
    double *Dh = (double *)xcalloc((size_t)pr->max_nodal_itr + 1, sizeof(double));
    int32_t ran = 0;
    for (itr = 0; itr < pr->max_nodal_itr; ++itr) {
        double D = 0.0;
        for (k = 0; k < nb; ++k) {
            int32_t first = k * bs, last = first + bs;
            if (last > V) last = V;
            if (first >= last) continue;
            D += mcmc_batch(st, pr, outer, (uint32_t)itr, first, last - first, stats);
        }
        Dh[itr] = D;
        if (D_out) D_out[itr] = D;
        ran = itr + 1;
        if (itr >= pr->window - 1 &&
            mcmc_converged(Dh, itr, pr->window, thresh, orc_mdl_of(st, pr->model_term, NULL)))
            break;
    }
    free(Dh);
    return ran;
}

/* The stopping rule alone against given per-iteration D[] and MDL[] (mock; no
 * MCMC): the number of iterations mcmc_phase would run (at most n). */
int32_t orc_mcmc_stop_mock(const double *D, const double *mdl, int32_t n, int32_t window, double thresh)
{
    int32_t itr;
    for (itr = 0; itr < n; ++itr)
        if (mcmc_converged(D, itr, window, thresh, mdl[itr])) return itr + 1;
    return n;
}

/*
 * Golden-section bracket update (P:34 1, Fig. 2, P:328 4.3; R:Z21;
 * GraphChallenge prepare_for_partition_on_next_num_blocks).  Slots hold
 * (b, B, MDL) ordered by B descending, slot 1 the best so far.  Stores the
 * round's (cur, B, S), then picks the next number of merges K and the slot to
 * restart from.  Returns 1 when the search is done (answer: slot 1).
 * sb may be NULL (mock runs: no partitions carried).
 */
static int bracket_step(int32_t **sb, int32_t *sB, double *sS, const int32_t *cur,
                        int32_t B, double S, int32_t V, double rate,
                        int32_t *K, int *restart)
{
    int idx;
    if (S <= sS[1]) {
        idx = (sB[1] > B) ? 0 : 2;
        if (sb) memcpy(sb[idx], sb[1], sizeof(int32_t) * (size_t)V);
        sB[idx] = sB[1];
        sS[idx] = sS[1];
        idx = 1;
    } else {
        idx = (sB[1] > B) ? 2 : 0;
    }
    if (sb) memcpy(sb[idx], cur, sizeof(int32_t) * (size_t)V);
    sB[idx] = B;
    sS[idx] = S;
    if (sS[2] == INFINITY) {
        *K = (int32_t)((double)B * rate);
        *restart = 1;
        return *K == 0;
    } else {
        int32_t next;
        if (sB[0] - sB[2] == 2) return 1;
        idx = ((sB[0] - sB[1]) >= (sB[1] - sB[2])) ? 0 : 1;
        next = sB[idx + 1] + (int32_t)nearbyint((double)(sB[idx] - sB[idx + 1]) * 0.618);
        *K = sB[idx] - next;
        *restart = idx;
        return *K <= 0;
    }
}

/* the bracket logic alone against a table MDL(B) (mock; no merging/MCMC):
 * starting from B = V, each round "merges" K blocks (B -> B - K) and scores
 * mdl_of_B[B].  Writes the visited B sequence; returns its length. */
int32_t orc_golden_mock(int32_t V, double rate, const double *mdl_of_B,
                        int32_t *visited, int32_t cap, int32_t *B_final)
{
    int32_t sB[3] = {0, 0, 0}, K, B = V, n = 0;
    double sS[3] = {INFINITY, INFINITY, INFINITY};
    int restart = 1;
    K = (int32_t)((double)B * rate);
    while (K > 0 && n < cap) {
        B = B - K;
        visited[n++] = B;
        if (bracket_step(NULL, sB, sS, NULL, B, mdl_of_B[B], V, rate, &K, &restart)) break;
        B = sB[restart];
    }
    if (B_final) *B_final = sB[1] ? sB[1] : V;
    return n;
}

/* The bracket logic replayed over a given sequence of rounds (B after the
 * merge, MDL of the round) -- e.g. another implementation's trace: for each
 * round k, the B the next round restarts from, its number of merges K
 * (bracket_step above) and whether the bracket is established after round k
 * (the next round then uses thresh2, R:Z19).  Returns the number of rounds
 * after which the search stops (n if it would go on). */
int32_t orc_bracket_replay(int32_t n, const int32_t *B, const double *S, double rate,
                           int32_t *Bstart_next, int32_t *K_next, int32_t *bracket_next)
{
    int32_t sB[3] = {0, 0, 0}, k, K = 0;
    double sS[3] = {INFINITY, INFINITY, INFINITY};
    int restart = 1;
    for (k = 0; k < n; ++k) {
        int done = bracket_step(NULL, sB, sS, NULL, B[k], S[k], 0, rate, &K, &restart);
        Bstart_next[k] = sB[restart];
        K_next[k] = K;
        bracket_next[k] = sS[2] != INFINITY;
        if (done) return k + 1;
    }
    return n;
}

/* trace rows (ORC_TRACE_COLS): [outer, B after merge, mcmc iterations, MDL,
 * convergence threshold used, accepted moves] per round */
#define ORC_TRACE_COLS 6
int32_t orc_partition(void *h, const OParams *pr, int32_t *b_out, int32_t *B_out,
                      double *mdl_out, OStats *stats, double *trace, int32_t trace_cap)
{
    OState *st = (OState *)h;
    int32_t V = st->g.V, i, K, rounds = 0;
    int32_t *sb[3];
    int32_t sB[3] = {0, 0, 0};
    double sS[3] = {INFINITY, INFINITY, INFINITY};
    uint32_t outer = 0;
    int done = 0;
    if (stats) memset(stats, 0, sizeof(*stats));
    for (i = 0; i < 3; ++i) sb[i] = (int32_t *)xcalloc((size_t)(V ? V : 1), sizeof(int32_t));
    for (i = 0; i < V; ++i) st->b[i] = i;
    st->B = V;
    rebuild(st);
    K = (int32_t)((double)st->B * pr->reduction_rate);
    if (K == 0) {
        /* nothing to merge: the singleton partition is the answer */
        sS[1] = orc_mdl_of(st, pr->model_term, NULL);
        sB[1] = st->B;
        memcpy(sb[1], st->b, sizeof(int32_t) * (size_t)V);
        done = 1;
    }
    while (!done && rounds < pr->max_rounds) {
        int bracket = (sS[2] != INFINITY);
        int32_t itrs, B;
        double S, thresh = bracket ? pr->thresh2 : pr->thresh1;
        int64_t acc0 = stats ? stats->n_move_acc : 0;
        merge_phase(st, pr, outer, K, stats);
        B = st->B;
        itrs = mcmc_phase(st, pr, outer, thresh, stats, NULL);
        S = orc_mdl_of(st, pr->model_term, NULL);
        if (trace && rounds < trace_cap) {
            double *row = trace + (size_t)ORC_TRACE_COLS * rounds;
            row[0] = (double)outer;
            row[1] = (double)B;
            row[2] = (double)itrs;
            row[3] = S;
            row[4] = thresh;
            row[5] = stats ? (double)(stats->n_move_acc - acc0) : 0.0;
        }
        if (stats) stats->mcmc_itr_total += itrs;
        ++rounds;
        {
            int idx = -1;
            int32_t *cur = st->b;
            if (bracket_step(sb, sB, sS, cur, B, S, V, pr->reduction_rate, &K, &idx)) {
                done = 1;
                break;
            }
            memcpy(st->b, sb[idx], sizeof(int32_t) * (size_t)V);
            st->B = sB[idx];
        }
        rebuild(st);
        ++outer;
    }
    /* the answer: the best slot */
    memcpy(st->b, sb[1], sizeof(int32_t) * (size_t)V);
    st->B = sB[1];
    rebuild(st);
    if (b_out) memcpy(b_out, st->b, sizeof(int32_t) * (size_t)V);
    if (B_out) *B_out = st->B;
    if (mdl_out) *mdl_out = sS[1];
    if (stats) stats->rounds = rounds;
    for (i = 0; i < 3; ++i) free(sb[i]);
    return rounds;
}

/* an MCMC phase alone from the current state (used by lockstep tests);
 * D_out: nullable, max_nodal_itr entries */
int32_t orc_mcmc_phase(void *h, const OParams *pr, uint32_t outer, double thresh, OStats *stats,
                       double *D_out)
{
    if (stats) memset(stats, 0, sizeof(*stats));
    return mcmc_phase((OState *)h, pr, outer, thresh, stats, D_out);
}

/* one merge phase alone from the current state */
int32_t orc_merge_phase(void *h, const OParams *pr, uint32_t outer, int32_t K)
{
    merge_phase((OState *)h, pr, outer, K, NULL);
    return ((OState *)h)->B;
}

/* one MCMC batch (snapshot, apply, rebuild) — returns the sum of accepted dS */
double orc_mcmc_batch(void *h, const OParams *pr, uint32_t outer, uint32_t itr,
                      int32_t first, int32_t count)
{
    return mcmc_batch((OState *)h, pr, outer, itr, first, count, NULL);
}
