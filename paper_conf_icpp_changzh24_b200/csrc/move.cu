// move.cu -- the vertex-move hot loop (P:141 3, P:176 3.2, P:238-246 3.3):
// for every vertex v of a batch, on the batch-start snapshot,
//   (a1) Philox proposal: weighted neighbour -> its block u -> uniform block
//        w.p. B/(B + d_u), else a weighted neighbour block of u (Alg. 1);
//   (a2) Delta S of moving v from r = b[v] to s (Eq. 7 in exact form), the
//        Hastings ratio and the Metropolis-Hastings decision.
//
// Delta S is decomposed over the unique neighbour blocks t of v (readings
// O.5, Z12, Z26): with o_t / i_t the out / in weight from v to block t
// (self-loop excluded, weight l):
//   dS = -sum_{t != r,s} [df(M_rt,-o_t) + df(M_st,o_t) + df(M_tr,-i_t) + df(M_ts,i_t)]
//        - [df(M_rr,-(o_r+i_r+l)) + df(M_rs,i_r-o_s) + df(M_sr,o_r-i_s) + df(M_ss,o_s+i_s+l)]
//        + df(dout_r,-kout) + df(dout_s,kout) + df(din_r,-kin) + df(din_s,kin)
// with df(m, d) = f(m + d) - f(m).  The (t, o_t, i_t) histogram is built in a
// shared-memory open-addressing table (one per warp; one per CTA for vertices
// whose neighbour-block count can exceed 128).  Each unique t is "owned" by
// its first adjacency position (atomicMin), and every thread sums the terms it
// owns in adjacency order, followed by a fixed shuffle tree: the result is
// deterministic and independent of the launch shape.
#include <algorithm>
#include <cstdlib>

#include "internal.h"
#include "prims.cuh"

namespace gsap {

constexpr int WARP_TAB = 256;          // slots per warp table (<= 128 keys)
constexpr int WARP_TAB_LOG2 = 8;
constexpr int BIG_THR = 128;           // warp path iff min(k_v, B) <= BIG_THR
constexpr int MOVE_WARPS = 8;          // warps per CTA, warp kernel
constexpr int CTA_THREADS = 256;       // big-vertex role: one CTA per vertex
constexpr int MID_TAB = 512;           // mid role: group tables (<= 256 keys)
#ifndef GSAP_MID_G
#define GSAP_MID_G 64
#endif
constexpr int MID_G = GSAP_MID_G;      // threads per mid-vertex group (64: four per CTA, 128: two)
constexpr int MID_PER_CTA = MOVE_WARPS * 32 / MID_G;
constexpr int MID_TAB_LOG2 = 9;
constexpr int CTA_SMEM_SLOTS = MOVE_WARPS * WARP_TAB;   // big-vertex shared table (<= 1024 keys)
constexpr size_t MOVE_SMEM = sizeof(int4) * MOVE_WARPS * WARP_TAB + sizeof(int) * MOVE_WARPS * (WARP_TAB / 2);
// vertices with > 1024 adjacency entries take the huge role (global tables when B > 1024)
#ifndef GSAP_MOVE_MINB
#define GSAP_MOVE_MINB 3               // CTAs per SM the register budget is sized for
#endif      // CTAs of the big-vertex role (grid-stride)

struct MoveArgs {
    int B;
    uint64_t seed;
    uint32_t outer, itr;
    const unsigned *itr_ptr;        // if set, the iteration is read from the device
    double beta;
    const int *__restrict__ rowptr, *__restrict__ col, *__restrict__ wgt;
    const int *__restrict__ cscptr, *__restrict__ cscsrc, *__restrict__ cscwgt;
    const int *__restrict__ kout, *__restrict__ kin, *__restrict__ selfw, *__restrict__ b;
    const int *__restrict__ nbo, *__restrict__ nbi;   // neighbour-block cache: b[col[p]], b[cscsrc[q]]
    BM m;
    int first, count;
    const int *__restrict__ list;   // big-vertex kernel: sorted vertex ids
    int list_count;
    int propose;                    // 1: k_move draws the proposal itself (MOVE_FUSED), else reads s_in
    const int *s_in;                // MOVE_DELTA
    int *s_out;
    double *dS, *H;
    unsigned char *acc;
    const int *__restrict__ mlist;  // mid vertices (128 < entries <= 256): 64-thread groups
    int mlist_count;
    int nmid_ctas;                  // CTAs [0, nmid_ctas): mid role (4 groups each)
    int big_log2;                   // big role: shared table of 2^big_log2 slots
    int nbig_ctas;                  // CTAs [0, nbig_ctas) take the big-vertex role
    const int *__restrict__ hlist;  // huge vertices (> 1024 adjacency entries), sorted ids
    int hlist_count;
    int4 *gtab;                     // huge role: global tables per CTA, or nullptr (shared)
    int gtab_log2;
    int nhuge_ctas;                 // CTAs [nbig_ctas, nbig_ctas + nhuge_ctas): huge role
    const int *__restrict__ perm;   // sorted two-pass mode: batch indices in line order
    double *part;                   // sorted two-pass mode: pass-1 partials, 3 per vertex
};

GSAP_DEV unsigned hash_slot(int t, int log2cap) {
    return ((unsigned)t * 0x9E3779B1u) >> (32 - log2cap);
}

GSAP_DEV int tab_insert(int4 *tab, int log2cap, int t) {
    const unsigned mask = (1u << log2cap) - 1u;
    unsigned sl = hash_slot(t, log2cap);
    while (true) {
        const int prev = atomicCAS(&tab[sl].x, -1, t);
        if (prev == -1 || prev == t) return (int)sl;
        sl = (sl + 1) & mask;
    }
}

// slot of key t, or -1 if absent
GSAP_DEV int tab_find(const int4 *tab, int log2cap, int t) {
    const unsigned mask = (1u << log2cap) - 1u;
    unsigned sl = hash_slot(t, log2cap);
    while (true) {
        const int k = *((volatile const int *)&tab[sl].x);
        if (k == t) return (int)sl;
        if (k == -1) return -1;
        sl = (sl + 1) & mask;
    }
}

// group-wide sums of three values (deterministic fixed trees)
// barrier of a G-thread group (G = 32: the warp; 256: the CTA; 64: one of
// four named-barrier groups of the CTA)
template <int G>
GSAP_DEV void gsync() {
    if (G == 32) __syncwarp();
    else if (G == 256) __syncthreads();
    else asm volatile("bar.sync %0, %1;" ::"r"(1 + (int)(threadIdx.x / G)), "r"(G) : "memory");
}

// group-wide sums of three values (deterministic fixed trees); sh: 3 G/32
// doubles owned by this group
template <int G>
GSAP_DEV void group_sum3(double &x, double &y, double &z, double *sh) {
    x = warp_sum(x);
    y = warp_sum(y);
    z = warp_sum(z);
    if (G == 32) return;
    const int w = (threadIdx.x % G) >> 5, lane = threadIdx.x & 31;
    if (lane == 0) {
        sh[w] = x;
        sh[G / 32 + w] = y;
        sh[2 * (G / 32) + w] = z;
    }
    gsync<G>();
    double a = 0.0, b = 0.0, c = 0.0;
#pragma unroll
    for (int i = 0; i < G / 32; ++i) {
        a += sh[i];
        b += sh[G / 32 + i];
        c += sh[2 * (G / 32) + i];
    }
    gsync<G>();
    x = a;
    y = b;
    z = c;
}


// sparse regime: four lookups (line k, key y_k) as interleaved branchless
// binary searches -- each step issues four independent loads, so a lane's
// dependent-load depth is log2(max len) + 1 instead of four times that
// (the lines of M live in HBM once the blockmodel outgrows L2)
#ifndef GSAP_LOOKUP_CONDCNT
#define GSAP_LOOKUP_CONDCNT 0
#endif
template <int N>
GSAP_DEV bool any_open(const int (&n)[N]) {
    bool o = false;
#pragma unroll
    for (int k = 0; k < N; ++k) o = o || n[k] > 1;
    return o;
}

template <int N>
GSAP_DEV void lookup4_in(const Line (&L)[N], const int (&y)[N], int (&p)[N], int (&n)[N], int (&out)[N]) {
    bool some[N];
#pragma unroll
    for (int k = 0; k < N; ++k) some[k] = n[k] > 0;
    while (any_open<N>(n)) {
#pragma unroll
        for (int k = 0; k < N; ++k) {
            if (n[k] > 1) {
                const int h = n[k] >> 1;
                p[k] = __ldg(L[k].idx + p[k] + h) <= y[k] ? p[k] + h : p[k];
                n[k] -= h;
            }
        }
    }
#pragma unroll
    for (int k = 0; k < N; ++k) {
        int v = 0;
        if (some[k]) {
#if GSAP_LOOKUP_CONDCNT
            // the count's sector only for a hit (one more dependent level)
            if (__ldg(L[k].idx + p[k]) == y[k]) v = __ldg(L[k].cnt + p[k]);
#else
            const int id = __ldg(L[k].idx + p[k]), cn = __ldg(L[k].cnt + p[k]);
            v = id == y[k] ? cn : 0;
#endif
        }
        out[k] = v;
    }
}

GSAP_DEV void lookup4(const Line (&L)[4], const int (&y)[4], int (&out)[4]) {
    int p[4] = {0, 0, 0, 0}, n[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) n[k] = L[k].len;
    lookup4_in(L, y, p, n, out);
}

// warp path, sparse regime: the 32 lanes of a vertex's warp all search the
// same four lines, so they first load 32 splitters per line together (lane j:
// idx[(j len) >> 5], one load level); a lane narrows each key to one of the 32
// buckets with five shuffles and binary-searches only that bucket -- five
// dependent load levels fewer per lookup once lines exceed 32 entries
template <int N>
GSAP_DEV void split4_load(const Line (&L)[N], int lane, int (&sp)[N]) {
#pragma unroll
    for (int k = 0; k < N; ++k) sp[k] = L[k].len > 0 ? __ldg(L[k].idx + ((lane * L[k].len) >> 5)) : 0x7fffffff;
}

// all 32 lanes: the bucket [p, p + n) of line k that holds key y[k] if present
// (n = 0: absent); sp[k] are line k's splitters as split4_load left them
template <int N>
GSAP_DEV void split4_bucket(const Line (&L)[N], const int (&sp)[N], const int (&y)[N], int (&p)[N], int (&n)[N]) {
#pragma unroll
    for (int k = 0; k < N; ++k) {
        int j = 0;   // the last bucket whose first entry is <= y[k]
#pragma unroll
        for (int st = 16; st >= 1; st >>= 1) {
            const int x = __shfl_sync(0xffffffffu, sp[k], j + st);
            if (x <= y[k]) j += st;
        }
        const int s0 = __shfl_sync(0xffffffffu, sp[k], 0);
        const int len = L[k].len, lo = (j * len) >> 5;
        p[k] = lo;
        n[k] = (len > 0 && s0 <= y[k]) ? (((j + 1) * len) >> 5) - lo : 0;
    }
}

// the state of one move r -> s that every term needs
struct MoveCtx {
    int v, r, s;
    long long Mrr, Mrs, Msr, Mss, o_r, i_r, o_s, i_s, kout, kin, l, dr, ds, Mrr2, Mrs2, Msr2, dr2, ds2;
    double Bd;
    Line Rr, Rs, Cr, Cs;
};

// dS / Hastings terms of one unique neighbour block t (out weight ot, in weight it)
GSAP_DEV void t_terms(const MoveArgs &a, const MoveCtx &q, int t, long long ot, long long it, double &accS,
                      double &pf, double &pb) {
    const double2 *__restrict__ ft = a.m.ft;
    const double *__restrict__ rcp = a.m.rcp;
    const double c = (double)(ot + it);
    if (t == q.r) {
        pf += c * (double)(q.Mrs + q.Msr + 1) * __ldg(rcp + q.r);
        pb += c * (double)(2 * q.Mrr2 + 1) / ((double)q.dr2 + q.Bd);
    } else if (t == q.s) {
        pf += c * (double)(2 * q.Mss + 1) * __ldg(rcp + q.s);
        pb += c * (double)(q.Msr2 + q.Mrs2 + 1) / ((double)q.ds2 + q.Bd);
    } else {
        long long Mrt, Mst, Mtr, Mts;
        if (a.m.dense) {
            Mrt = row_at(a.m, q.Rr, q.r, t);
            Mst = row_at(a.m, q.Rs, q.s, t);
            Mtr = col_at(a.m, q.Cr, q.r, t);
            Mts = col_at(a.m, q.Cs, q.s, t);
        } else {
            const Line Ln[4] = {q.Rr, q.Rs, q.Cr, q.Cs};
            const int yt[4] = {t, t, t, t};
            int o4[4];
            lookup4(Ln, yt, o4);
            Mrt = o4[0];
            Mst = o4[1];
            Mtr = o4[2];
            Mts = o4[3];
        }
        const double rt = __ldg(rcp + t);
        accS -= df_t(ft, Mrt, -ot) + df_t(ft, Mst, ot) + df_t(ft, Mtr, -it) + df_t(ft, Mts, it);
        pf += c * (double)(Mts + Mst + 1) * rt;
        pb += c * (double)(Mtr - it + Mrt - ot + 1) * rt;
    }
}

// the 2x2 core, the four degree terms and the two self-loop terms: term k of 10
GSAP_DEV void core_term(const MoveArgs &a, const MoveCtx &q, int k, double &accS, double &pf, double &pb) {
    const double2 *__restrict__ ft = a.m.ft;
    switch (k) {
        case 0: accS -= df_t(ft, q.Mrr, -(q.o_r + q.i_r + q.l)); break;
        case 1: accS -= df_t(ft, q.Mrs, q.i_r - q.o_s); break;
        case 2: accS -= df_t(ft, q.Msr, q.o_r - q.i_s); break;
        case 3: accS -= df_t(ft, q.Mss, q.o_s + q.i_s + q.l); break;
        case 4: accS += df_t(ft, __ldg(a.m.dout + q.r), -q.kout); break;
        case 5: accS += df_t(ft, __ldg(a.m.dout + q.s), q.kout); break;
        case 6: accS += df_t(ft, __ldg(a.m.din + q.r), -q.kin); break;
        case 7: accS += df_t(ft, __ldg(a.m.din + q.s), q.kin); break;
        case 8:
            if (q.l > 0) pf += 2.0 * (double)q.l * (double)(q.Mrs + q.Msr + 1) * __ldg(a.m.rcp + q.r);
            break;
        default:
            if (q.l > 0) pb += 2.0 * (double)q.l * (double)(q.Msr2 + q.Mrs2 + 1) / ((double)q.ds2 + q.Bd);
            break;
    }
}

// after phase A: the core values (every thread, redundantly: broadcast loads)
GSAP_DEV void move_ctx(const MoveArgs &a, int v, int r, int s, const int4 *tab, int log2cap, MoveCtx &q) {
    q.v = v;
    q.r = r;
    q.s = s;
    if (!a.m.dense) {
        q.Rr = row_line(a.m, r);
        q.Rs = row_line(a.m, s);
        q.Cr = col_line(a.m, r);
        q.Cs = col_line(a.m, s);
    }
    if (a.m.dense) {
        q.Mrr = row_at(a.m, q.Rr, r, r);
        q.Mrs = row_at(a.m, q.Rr, r, s);
        q.Msr = row_at(a.m, q.Rs, s, r);
        q.Mss = row_at(a.m, q.Rs, s, s);
    } else {
        const Line Lc[4] = {q.Rr, q.Rr, q.Rs, q.Rs};
        const int yc[4] = {r, s, r, s};
        int oc[4];
        lookup4(Lc, yc, oc);
        q.Mrr = oc[0];
        q.Mrs = oc[1];
        q.Msr = oc[2];
        q.Mss = oc[3];
    }
    const int slr = tab_find(tab, log2cap, r), sls = tab_find(tab, log2cap, s);
    q.o_r = slr >= 0 ? tab[slr].y : 0;
    q.i_r = slr >= 0 ? tab[slr].z : 0;
    q.o_s = sls >= 0 ? tab[sls].y : 0;
    q.i_s = sls >= 0 ? tab[sls].z : 0;
    q.kout = __ldg(a.kout + v);
    q.kin = __ldg(a.kin + v);
    q.l = __ldg(a.selfw + v);
    q.dr = bm_deg(a.m, r);
    q.ds = bm_deg(a.m, s);
    q.Mrr2 = q.Mrr - q.o_r - q.i_r - q.l;
    q.Mrs2 = q.Mrs + q.i_r - q.o_s;
    q.Msr2 = q.Msr + q.o_r - q.i_s;
    q.dr2 = q.dr - q.kout - q.kin;
    q.ds2 = q.ds + q.kout + q.kin;
    q.Bd = (double)a.B;
}

GSAP_DEV void mh_decide(const MoveArgs &a, const MoveCtx &q, uint4 w, double dS, double pf, double pb,
                        double &dS_out, double &H_out, bool &acc_out) {
    const double H = (q.kout + q.kin == 0) ? 1.0 : pb / pf;
    const double p = exp(-a.beta * dS) * H;
    const double u = ((double)w.w + 0.5) * (1.0 / 4294967296.0);
    dS_out = dS;
    H_out = H;
    acc_out = u <= p;
}

// the block of v's adjacency entry j (out-CSR entries first, then in-CSC),
// from the neighbour-block cache (no gather of b)
GSAP_DEV int nb_block(const MoveArgs &a, int ro, int nout, int ci, int j) {
    return j < nout ? __ldg(a.nbo + ro + j) : __ldg(a.nbi + ci + (j - nout));
}

// whether v's adjacency entry j is its self-loop: the neighbour ids are read
// only for vertices that have one (selfw[v] > 0), the others never load them
GSAP_DEV bool nb_self(const MoveArgs &a, int v, bool has_self, int ro, int nout, int ci, int j) {
    if (!has_self) return false;
    return (j < nout ? __ldg(a.col + ro + j) : __ldg(a.cscsrc + ci + (j - nout))) == v;
}

// (a1) one thread per vertex: the proposal chain is a handful of dependent
// loads, so 32 vertices per warp keep them in flight (R:O.4).
template <bool WEIGHTED>
GSAP_DEV int propose_move_thread(const MoveArgs &a, int v, uint4 w) {
    const uint32_t B = (uint32_t)a.B;
    const uint32_t K = (uint32_t)(__ldg(a.kout + v) + __ldg(a.kin + v));
    if (K == 0) return (int)pick(w.z, B);
    const int ro = __ldg(a.rowptr + v), nout = __ldg(a.rowptr + v + 1) - ro;
    const int ci = __ldg(a.cscptr + v);
    const uint32_t p = pick(w.x, K);
    int j;   // the chosen adjacency entry (out entries, then in entries)
    if (!WEIGHTED) {
        j = (int)p;
    } else {
        long long acc = 0;
        j = -1;
        for (int e = 0; e < nout && j < 0; ++e) {
            acc += __ldg(a.wgt + ro + e);
            if ((long long)p < acc) j = e;
        }
        const int nin = __ldg(a.cscptr + v + 1) - ci;
        for (int e = 0; e < nin && j < 0; ++e) {
            acc += __ldg(a.cscwgt + ci + e);
            if ((long long)p < acc) j = nout + e;
        }
    }
    const int u = nb_block(a, ro, nout, ci, j);
    const uint32_t du = (uint32_t)bm_deg(a.m, u);
    if (coin_random(w.y, B, du)) return (int)pick(w.z, B);
    if (a.m.mt) return __ldg(a.m.mt + u);   // N4: the shared table entry of u (Alg. 1 line 10)
    return bm_walk(a.m, u, (long long)pick(w.z, du), -1);
}

// the proposal of a warp-path vertex (R:O.4, Alg. 1): the neighbour at
// position p and its block come from the adjacency registers (nb, tb: entry
// 32 c + lane in nb[c]) when p < 128 in an unweighted graph; the walk over
// row / column u is a 32-ary warp search.  Same integer result as
// propose_move_thread.
template <bool WEIGHTED>
GSAP_DEV int propose_warp(const MoveArgs &a, int v, uint4 w, int deg, const int (&tb)[4]) {
    const uint32_t B = (uint32_t)a.B;
    if (WEIGHTED || deg > 128) return propose_move_thread<WEIGHTED>(a, v, w);   // warp-uniform
    if (deg == 0) return (int)pick(w.z, B);
    const uint32_t p = pick(w.x, (uint32_t)deg);
    const int c = (int)(p >> 5);
    const int x = c == 0 ? tb[0] : c == 1 ? tb[1] : c == 2 ? tb[2] : tb[3];
    const int u = __shfl_sync(FULL, x, (int)(p & 31u));
    const uint32_t du = (uint32_t)bm_deg(a.m, u);
    if (coin_random(w.y, B, du)) return (int)pick(w.z, B);
    if (a.m.mt) return __ldg(a.m.mt + u);   // N4
    return bm_walk_warp(a.m, u, (long long)pick(w.z, du));
}

// (a1 + a2), one warp per vertex (at most 128 adjacency entries, or B <= 128):
// adjacency ids and their blocks are loaded once into registers and serve
// both the proposal and the neighbour-block histogram; phase A builds the
// shared-memory table and compacts the unique blocks into `list` in
// first-occurrence order; phase B gives each lane whole unique blocks.  The
// 2x2 core and the four degree terms take lanes 0..7 with one df each.
// int32 throughout (weights and counts < 2^30, gsap.h).  Table left empty.
template <bool WEIGHTED, bool DENSE>
GSAP_DEV void move_vertex_warp(const MoveArgs &a, int i, int4 *tab, int *list) {
    const int lane = threadIdx.x & 31;
    const unsigned lt = (1u << lane) - 1u;
    const int v = a.first + i;
    const int ro = __ldg(a.rowptr + v), nout = __ldg(a.rowptr + v + 1) - ro;
    const int ci = __ldg(a.cscptr + v), nin = __ldg(a.cscptr + v + 1) - ci;
    const int deg = nout + nin;
    const bool has_self = __ldg(a.selfw + v) > 0;
    int tb[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) {   // the neighbours' blocks, from the cache (no gather of b)
        const int j = c * 32 + lane;
        tb[c] = j < deg ? nb_block(a, ro, nout, ci, j) : -1;
    }
    bool self[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) self[c] = c * 32 + lane < deg && nb_self(a, v, has_self, ro, nout, ci, c * 32 + lane);
    const int r = __ldg(a.b + v);
    const uint32_t itr = a.itr_ptr ? __ldg(a.itr_ptr) : a.itr;
    const uint4 w = draws(a.seed, (uint32_t)v, 0u, itr, a.outer, 1u);
    const int B = a.m.B;
    // ---- (a1) first half of the proposal (R:O.4): the neighbour's block u
    // comes from the adjacency registers; every load the walk over row /
    // column u needs is issued now, so it overlaps the histogram below
    const bool fast = a.propose && !WEIGHTED && deg <= 128 && deg > 0;
    int u = 0, dout_u = 0, din_u = 0, rlo = 0, rhi = 0, clo = 0, chi = 0;
    if (fast) {
        const uint32_t p = pick(w.x, (uint32_t)deg);
        const int c = (int)(p >> 5);
        const int x = c == 0 ? tb[0] : c == 1 ? tb[1] : c == 2 ? tb[2] : tb[3];
        u = __shfl_sync(FULL, x, (int)(p & 31u));
        dout_u = __ldg(a.m.dout + u);
        din_u = __ldg(a.m.din + u);
        rlo = __ldg(a.m.rowptr + u);
        rhi = __ldg(a.m.rowend + u);
        clo = __ldg(a.m.colptr + u);
        chi = __ldg(a.m.colend + u);
    }
    // ---- phase A: histogram of v's neighbour blocks (self-loop excluded),
    // independent of the proposal; unique blocks compacted into `list`
    int keep[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        keep[c] = -1;
        const int j = c * 32 + lane;
        if (tb[c] >= 0 && !self[c]) {
            const bool out = j < nout;
            const int wt = WEIGHTED ? (out ? __ldg(a.wgt + ro + j) : __ldg(a.cscwgt + ci + j - nout)) : 1;
            const int sl = tab_insert(tab, WARP_TAB_LOG2, tb[c]);
            atomicAdd(out ? &tab[sl].y : &tab[sl].z, wt);
            atomicMin(&tab[sl].w, j);
            keep[c] = sl;
        }
    }
    for (int j = 128 + lane; j < deg; j += 32) {   // only when B <= 128 (<= B keys)
        const bool out = j < nout;
        if (nb_self(a, v, has_self, ro, nout, ci, j)) continue;
        const int wt = WEIGHTED ? (out ? __ldg(a.wgt + ro + j) : __ldg(a.cscwgt + ci + j - nout)) : 1;
        const int sl = tab_insert(tab, WARP_TAB_LOG2, nb_block(a, ro, nout, ci, j));
        atomicAdd(out ? &tab[sl].y : &tab[sl].z, wt);
        atomicMin(&tab[sl].w, j);
    }
    __syncwarp();
    int nuniq = 0;
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        const int sl = keep[c];
        const bool own = sl >= 0 && tab[sl].w == c * 32 + lane;
        const unsigned bal = __ballot_sync(FULL, own);
        if (own) list[nuniq + __popc(bal & lt)] = sl;
        nuniq += __popc(bal);
    }
    for (int base = 128; base < deg; base += 32) {
        const int j = base + lane;
        int sl = -1;
        if (j < deg && !nb_self(a, v, has_self, ro, nout, ci, j))
            sl = tab_find(tab, WARP_TAB_LOG2, nb_block(a, ro, nout, ci, j));
        const bool own = sl >= 0 && tab[sl].w == j;
        const unsigned bal = __ballot_sync(FULL, own);
        if (own) list[nuniq + __popc(bal & lt)] = sl;
        nuniq += __popc(bal);
    }
    __syncwarp();
    // r-side entries of this lane's first unique block (dense regime), also
    // independent of the proposal
    int4 e0 = make_int4(-1, 0, 0, 0);
    int Mrt0 = 0, Mtr0 = 0;
    double rt0 = 0.0;
    const int *__restrict__ D = a.m.dense;   // non-null iff DENSE
    if (lane < nuniq) {
        e0 = tab[list[lane]];
        if (DENSE) {
            Mrt0 = __ldg(D + (size_t)r * B + e0.x);
            Mtr0 = __ldg(D + (size_t)e0.x * B + r);
            rt0 = __ldg(a.m.rcp + e0.x);
        }
    }
    // ---- (a1) second half: coin, then the walk
    int s;
    if (!a.propose) {
        s = a.s_in[i];
    } else if (fast) {
        const uint32_t du = (uint32_t)(dout_u + din_u);
        if (coin_random(w.y, (uint32_t)B, du)) {
            s = (int)pick(w.z, (uint32_t)B);
        } else if (a.m.mt) {
            s = __ldg(a.m.mt + u);   // N4: the shared table entry of u (Alg. 1 line 10)
        } else {
            const long long q = (long long)pick(w.z, du);
            if (q < dout_u) s = __ldg(a.m.col + warp_upper_bound(a.m.cum, rlo, rhi, q));
            else s = __ldg(a.m.row + warp_upper_bound(a.m.ccum, clo, chi, q - dout_u));
        }
    } else {
        s = propose_warp<WEIGHTED>(a, v, w, deg, tb);
    }
    if (a.propose && lane == 0) a.s_out[i] = s;
    double dS = 0.0, H = 1.0;
    bool acc = false;
    if (s != r) {
        // ---- core state
        const int slr = tab_find(tab, WARP_TAB_LOG2, r), sls = tab_find(tab, WARP_TAB_LOG2, s);
        const int o_r = slr >= 0 ? tab[slr].y : 0, i_r = slr >= 0 ? tab[slr].z : 0;
        const int o_s = sls >= 0 ? tab[sls].y : 0, i_s = sls >= 0 ? tab[sls].z : 0;
        const int kout = __ldg(a.kout + v), kin = __ldg(a.kin + v), l = __ldg(a.selfw + v);
        const int dout_r = __ldg(a.m.dout + r), dout_s = __ldg(a.m.dout + s);
        const int din_r = __ldg(a.m.din + r), din_s = __ldg(a.m.din + s);
        int Mrr, Mrs, Msr, Mss;
        Line Ln[4];   // sparse: row r, row s, column r, column s of M
        int sp[4];    // sparse: this lane's splitter of each of the four lines
        if (DENSE) {
            Mrr = __ldg(D + (size_t)r * B + r);
            Mrs = __ldg(D + (size_t)r * B + s);
            Msr = __ldg(D + (size_t)s * B + r);
            Mss = __ldg(D + (size_t)s * B + s);
        } else {
            Ln[0] = row_line(a.m, r);
            Ln[1] = row_line(a.m, s);
            Ln[2] = col_line(a.m, r);
            Ln[3] = col_line(a.m, s);
            split4_load(Ln, lane, sp);
            const Line Lc[4] = {Ln[0], Ln[0], Ln[1], Ln[1]};
            const int spc[4] = {sp[0], sp[0], sp[1], sp[1]};
            const int yc[4] = {r, s, r, s};
            int oc[4], pc[4], nc[4];
            split4_bucket(Lc, spc, yc, pc, nc);
            lookup4_in(Lc, yc, pc, nc, oc);
            Mrr = oc[0];
            Mrs = oc[1];
            Msr = oc[2];
            Mss = oc[3];
        }
        const double Bd = (double)B;
        const int Mrr2 = Mrr - o_r - i_r - l, Mrs2 = Mrs + i_r - o_s, Msr2 = Msr + o_r - i_s;
        const int dr2 = dout_r + din_r - kout - kin, ds2 = dout_s + din_s + kout + kin;
        const double2 *__restrict__ ft = a.m.ft;
        const double *__restrict__ rcp = a.m.rcp;
        // ---- phase B: one unique neighbour block per lane
        double accS = 0.0, pf = 0.0, pb = 0.0;
        for (int base = 0; base < nuniq; base += 32) {   // warp-uniform trips (shuffles below)
            const int k = base + lane;
            const int4 e = k >= nuniq ? make_int4(-1, 0, 0, 0) : k == lane ? e0 : tab[list[k]];
            const int t = e.x, ot = e.y, it = e.z;
            int pb4[4], nb4[4];
            if (!DENSE) {
                const int yt[4] = {t, t, t, t};
                split4_bucket(Ln, sp, yt, pb4, nb4);
            }
            if (k >= nuniq) continue;
            const double cw = (double)(ot + it);
            if (t == r) {
                pf += cw * (double)(Mrs + Msr + 1) * __ldg(rcp + r);
                pb += cw * (double)(2 * Mrr2 + 1) / ((double)dr2 + Bd);
            } else if (t == s) {
                pf += cw * (double)(2 * Mss + 1) * __ldg(rcp + s);
                pb += cw * (double)(Msr2 + Mrs2 + 1) / ((double)ds2 + Bd);
            } else {
                int Mrt, Mst, Mtr, Mts;
                double rt;
                if (DENSE) {
                    if (k == lane) {
                        Mrt = Mrt0;
                        Mtr = Mtr0;
                        rt = rt0;
                    } else {
                        Mrt = __ldg(D + (size_t)r * B + t);
                        Mtr = __ldg(D + (size_t)t * B + r);
                        rt = __ldg(rcp + t);
                    }
                    Mst = __ldg(D + (size_t)s * B + t);
                    Mts = __ldg(D + (size_t)t * B + s);
                } else {
                    const int yt[4] = {t, t, t, t};
                    int o4[4];
                    lookup4_in(Ln, yt, pb4, nb4, o4);
                    Mrt = o4[0];
                    Mst = o4[1];
                    Mtr = o4[2];
                    Mts = o4[3];
                    rt = __ldg(rcp + t);
                }
                accS -= df_t(ft, Mrt, -ot) + df_t(ft, Mst, ot) + df_t(ft, Mtr, -it) + df_t(ft, Mts, it);
                pf += cw * (double)(Mts + Mst + 1) * rt;
                pb += cw * (double)(Mtr - it + Mrt - ot + 1) * rt;
            }
        }
        // the 2x2 core (lanes 0..3) and the degree terms (lanes 4..7), one df each
        if (lane < 8) {
            const int m = lane == 0 ? Mrr : lane == 1 ? Mrs : lane == 2 ? Msr : lane == 3 ? Mss
                        : lane == 4 ? dout_r : lane == 5 ? dout_s : lane == 6 ? din_r : din_s;
            const int d = lane == 0 ? -(o_r + i_r + l) : lane == 1 ? i_r - o_s : lane == 2 ? o_r - i_s
                        : lane == 3 ? o_s + i_s + l : lane == 4 ? -kout : lane == 5 ? kout : lane == 6 ? -kin : kin;
            const double x = df_t(ft, m, d);
            accS += lane < 4 ? -x : x;
        }
        if (lane == 0 && l > 0) {   // v's self-loop in the forward / backward proposal laws (R:Z26)
            pf += 2.0 * (double)l * (double)(Mrs + Msr + 1) * __ldg(rcp + r);
            pb += 2.0 * (double)l * (double)(Msr2 + Mrs2 + 1) / ((double)ds2 + Bd);
        }
        accS = warp_sum(accS);
        pf = warp_sum(pf);
        pb = warp_sum(pb);
        dS = accS;
        H = (kout + kin == 0) ? 1.0 : pb / pf;
        const double p = exp(-a.beta * dS) * H;
        acc = ((double)w.w + 0.5) * (1.0 / 4294967296.0) <= p;
    }
    // leave the table empty: exactly the listed slots were used (after every
    // lane's last table read: the shuffles above converge the warp but do not
    // order shared memory, __syncwarp does)
    __syncwarp();
    for (int k = lane; k < nuniq; k += 32) tab[list[k]] = make_int4(-1, 0, 0, 0x7fffffff);
    __syncwarp();
    if (lane == 0) {
        if (a.dS) a.dS[i] = dS;
        if (a.H) a.H[i] = H;
        if (a.acc) a.acc[i] = acc ? 1 : 0;
    }
}

// ------------------------------------------------------ sorted two-pass --
// Large sparse blockmodels (lines of M far outside L2): a vertex move reads
// four lines of M (rows and columns r and s), and lines fetched per vertex
// are fetched again by the next vertex of the same block.  Here the batch is
// evaluated in two passes over the SAME snapshot, each visiting the vertices
// grouped by one of its two blocks (counting sort of the batch by r = b[v] and
// by the proposal s), so consecutive warps search the same two lines and a
// line leaves HBM about once per block and pass:
//   pass 1 (grouped by r): rows / columns r -- every dS / Hastings term that
//     reads M_r. or M_.r, the 2x2 core entries M_rr, M_rs, M_sr, the degree
//     terms and the whole backward law p_bwd (R:Z26);
//   pass 2 (grouped by s): rows / columns s -- the terms in M_s. / M_.s and
//     M_ss, then dS, H = p_bwd / p_fwd and the MH decision (Eq. 7, R:O.5).
// The split follows the decomposition above term by term; only the order of
// the floating-point sums differs from the fused kernel.  Vertices with more
// than 128 adjacency entries stay in k_move_groups (fused terms, s given).
// wide splitters: K per lane (32 K per line, lane l holds splitters l K ..
// l K + K - 1: entry floor(g len / (32 K)) for splitter g); a key's bucket is
// found with 5 + (K - 1) shuffles and holds <= ceil(len / (32 K)) entries,
// which are then scanned with independent loads (one memory round for
// lines of <= 256 K entries instead of a dependent binary search)
template <int N, int K>
GSAP_DEV void splitw_load(const Line (&L)[N], int lane, int (&sp)[N][K]) {
#pragma unroll
    for (int k = 0; k < N; ++k)
#pragma unroll
        for (int e = 0; e < K; ++e)
            sp[k][e] = L[k].len > 0 ? __ldg(L[k].idx + (int)(((long long)(lane * K + e) * L[k].len) / (32 * K)))
                                    : 0x7fffffff;
}

template <int N, int K>
GSAP_DEV void splitw_bucket(const Line (&L)[N], const int (&sp)[N][K], const int (&y)[N], int (&p)[N],
                            int (&n)[N]) {
#pragma unroll
    for (int k = 0; k < N; ++k) {
        int j = 0;   // the last lane whose first splitter is <= y[k]
#pragma unroll
        for (int st = 16; st >= 1; st >>= 1) {
            const int x = __shfl_sync(0xffffffffu, sp[k][0], j + st);
            if (x <= y[k]) j += st;
        }
        int e = 0;   // the last of lane j's splitters <= y[k]
#pragma unroll
        for (int q = 1; q < K; ++q) {
            const int x = __shfl_sync(0xffffffffu, sp[k][q], j);
            if (x <= y[k]) e = q;
        }
        const int s0 = __shfl_sync(0xffffffffu, sp[k][0], 0);
        const int len = L[k].len, g = j * K + e;
        const int lo = (int)(((long long)g * len) / (32 * K)), hi = (int)(((long long)(g + 1) * len) / (32 * K));
        p[k] = lo;
        n[k] = (len > 0 && s0 <= y[k]) ? hi - lo : 0;
    }
}

// M entry of key y[k] in bucket [p[k], p[k] + n[k]) of line k: binary
// search down to <= W entries, then up to W independent id loads; the count
// only on a hit (W = 8 for 128 splitters per line, 4 for 256: the bucket of a
// line of <= 1024 entries never needs the search)
template <int N, int W = 8>
GSAP_DEV void bucket_get(const Line (&L)[N], const int (&y)[N], int (&p)[N], int (&n)[N], int (&out)[N]) {
#pragma unroll
    for (int k = 0; k < N; ++k) {
        while (n[k] > W) {
            const int h = n[k] >> 1;
            p[k] = __ldg(L[k].idx + p[k] + h) <= y[k] ? p[k] + h : p[k];
            n[k] -= h;
        }
    }
    int id[N][W];
#pragma unroll
    for (int k = 0; k < N; ++k)
#pragma unroll
        for (int q = 0; q < W; ++q) id[k][q] = q < n[k] ? __ldg(L[k].idx + p[k] + q) : -1;
#pragma unroll
    for (int k = 0; k < N; ++k) {
        int hit = -1;
#pragma unroll
        for (int q = 0; q < W; ++q) hit = id[k][q] == y[k] ? q : hit;
        out[k] = hit >= 0 ? __ldg(L[k].cnt + p[k] + hit) : 0;
    }
}

#ifndef GSAP_HALF_K
#define GSAP_HALF_K 4
#endif
constexpr int HALF_K = GSAP_HALF_K;   // splitters per lane in the sorted two-pass kernels
constexpr int HALF_W = HALF_K >= 8 ? 4 : 8;   // bucket scan width (bucket_get)

template <bool WEIGHTED, int PASS>
GSAP_DEV void move_vertex_half(const MoveArgs &a, int i, int4 *tab, int *list) {
    const int lane = threadIdx.x & 31;
    const unsigned lt = (1u << lane) - 1u;
    const int v = a.first + i;
    const int r = __ldg(a.b + v);
    const int s = a.s_in[i];
    if (s == r) {   // R:Z13 (warp-uniform)
        if (PASS == 2 && lane == 0) {
            if (a.dS) a.dS[i] = 0.0;
            if (a.H) a.H[i] = 1.0;
            if (a.acc) a.acc[i] = 0;
        }
        return;
    }
    const int ro = __ldg(a.rowptr + v), nout = __ldg(a.rowptr + v + 1) - ro;
    const int ci = __ldg(a.cscptr + v), nin = __ldg(a.cscptr + v + 1) - ci;
    const int deg = nout + nin;   // <= 128 (the caller routes bigger vertices to k_move_groups)
    const bool has_self = __ldg(a.selfw + v) > 0;
    const int B = a.m.B;
    // the two lines of this pass and their wide splitters (32 HALF_K per
    // line, shared by the warp), issued before the histogram
    Line Ln[2];
    const int x = PASS == 1 ? r : s;
    Ln[0] = row_line(a.m, x);
    Ln[1] = col_line(a.m, x);
    int sp[2][HALF_K];
    splitw_load<2, HALF_K>(Ln, lane, sp);
    // ---- phase A: histogram of v's neighbour blocks (self-loop excluded)
    int keep[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        keep[c] = -1;
        const int j = c * 32 + lane;
        if (j < deg) {
            const bool out = j < nout;
            if (!nb_self(a, v, has_self, ro, nout, ci, j)) {
                const int wt = WEIGHTED ? (out ? __ldg(a.wgt + ro + j) : __ldg(a.cscwgt + ci + j - nout)) : 1;
                const int sl = tab_insert(tab, WARP_TAB_LOG2, nb_block(a, ro, nout, ci, j));
                atomicAdd(out ? &tab[sl].y : &tab[sl].z, wt);
                atomicMin(&tab[sl].w, j);
                keep[c] = sl;
            }
        }
    }
    __syncwarp();
    int nuniq = 0;
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        const int sl = keep[c];
        const bool own = sl >= 0 && tab[sl].w == c * 32 + lane;
        const unsigned bal = __ballot_sync(FULL, own);
        if (own) list[nuniq + __popc(bal & lt)] = sl;
        nuniq += __popc(bal);
    }
    __syncwarp();
    const int slr = tab_find(tab, WARP_TAB_LOG2, r), sls = tab_find(tab, WARP_TAB_LOG2, s);
    const int o_r = slr >= 0 ? tab[slr].y : 0, i_r = slr >= 0 ? tab[slr].z : 0;
    const int o_s = sls >= 0 ? tab[sls].y : 0, i_s = sls >= 0 ? tab[sls].z : 0;
    const int kout = __ldg(a.kout + v), kin = __ldg(a.kin + v), l = __ldg(a.selfw + v);
    const int dout_r = __ldg(a.m.dout + r), dout_s = __ldg(a.m.dout + s);
    const int din_r = __ldg(a.m.din + r), din_s = __ldg(a.m.din + s);
    const double Bd = (double)B;
    const int dr2 = dout_r + din_r - kout - kin, ds2 = dout_s + din_s + kout + kin;
    const double2 *__restrict__ ft = a.m.ft;
    const double *__restrict__ rcp = a.m.rcp;
    // ---- core entries of this pass: pass 1 M_rr, M_rs (row r), M_sr (column r); pass 2 M_ss (row s)
    int Mrr = 0, Mrs = 0, Msr = 0, Mss = 0;
    if (PASS == 1) {   // row r at r and s, column r at s
        const Line Lc[3] = {Ln[0], Ln[0], Ln[1]};
        int spc[3][HALF_K];
#pragma unroll
        for (int e = 0; e < HALF_K; ++e) {
            spc[0][e] = sp[0][e];
            spc[1][e] = sp[0][e];
            spc[2][e] = sp[1][e];
        }
        const int yc[3] = {r, s, s};
        int pc[3], nc[3], oc[3];
        splitw_bucket<3, HALF_K>(Lc, spc, yc, pc, nc);
        bucket_get<3, HALF_W>(Lc, yc, pc, nc, oc);
        Mrr = oc[0];
        Mrs = oc[1];
        Msr = oc[2];
    } else {           // row s at s
        const Line Lc[1] = {Ln[0]};
        int spc[1][HALF_K];
#pragma unroll
        for (int e = 0; e < HALF_K; ++e) spc[0][e] = sp[0][e];
        const int yc[1] = {s};
        int pc[1], nc[1], oc[1];
        splitw_bucket<1, HALF_K>(Lc, spc, yc, pc, nc);
        bucket_get<1, HALF_W>(Lc, yc, pc, nc, oc);
        Mss = oc[0];
    }
    const int Mrr2 = Mrr - o_r - i_r - l, Mrs2 = Mrs + i_r - o_s, Msr2 = Msr + o_r - i_s;
    // ---- phase B: one unique neighbour block per lane, this pass's two lines
    double accS = 0.0, pf = 0.0, pb = 0.0;
    for (int base = 0; base < nuniq; base += 32) {   // warp-uniform trips (shuffles below)
        const int k = base + lane;
        const int4 e = k >= nuniq ? make_int4(-1, 0, 0, 0) : tab[list[k]];
        const int t = e.x, ot = e.y, it = e.z;
        int pb2[2], nb2[2];
        {
            const int yt[2] = {t, t};
            splitw_bucket<2, HALF_K>(Ln, sp, yt, pb2, nb2);
        }
        if (k >= nuniq) continue;
        const double cw = (double)(ot + it);
        if (t == r) {
            if (PASS == 1) {
                pf += cw * (double)(Mrs + Msr + 1) * __ldg(rcp + r);
                pb += cw * (double)(2 * Mrr2 + 1) / ((double)dr2 + Bd);
            }
        } else if (t == s) {
            if (PASS == 1) pb += cw * (double)(Msr2 + Mrs2 + 1) / ((double)ds2 + Bd);
            else pf += cw * (double)(2 * Mss + 1) * __ldg(rcp + s);
        } else {
            int o2[2];
            {
                const int yt[2] = {t, t};
                bucket_get<2, HALF_W>(Ln, yt, pb2, nb2, o2);
            }
            const double rt = __ldg(rcp + t);
            if (PASS == 1) {   // o2 = {M_rt, M_tr}
                accS -= df_t(ft, o2[0], -ot) + df_t(ft, o2[1], -it);
                pb += cw * (double)(o2[1] - it + o2[0] - ot + 1) * rt;
            } else {           // o2 = {M_st, M_ts}
                accS -= df_t(ft, o2[0], ot) + df_t(ft, o2[1], it);
                pf += cw * (double)(o2[1] + o2[0] + 1) * rt;
            }
        }
    }
    // the 2x2 core, the degree terms and v's self-loop in the proposal laws (R:Z26)
    if (PASS == 1) {
        if (lane < 7 && lane != 3) {
            const int m = lane == 0 ? Mrr : lane == 1 ? Mrs : lane == 2 ? Msr
                        : lane == 4 ? dout_r : lane == 5 ? dout_s : din_r;
            const int d = lane == 0 ? -(o_r + i_r + l) : lane == 1 ? i_r - o_s : lane == 2 ? o_r - i_s
                        : lane == 4 ? -kout : lane == 5 ? kout : -kin;
            const double y = df_t(ft, m, d);
            accS += lane < 4 ? -y : y;
        }
        if (lane == 7) accS += df_t(ft, din_s, kin);
        if (lane == 0 && l > 0) {
            pf += 2.0 * (double)l * (double)(Mrs + Msr + 1) * __ldg(rcp + r);
            pb += 2.0 * (double)l * (double)(Msr2 + Mrs2 + 1) / ((double)ds2 + Bd);
        }
    } else if (lane == 3) {
        accS -= df_t(ft, Mss, o_s + i_s + l);
    }
    accS = warp_sum(accS);
    pf = warp_sum(pf);
    if (PASS == 1) pb = warp_sum(pb);
    // leave the table empty: exactly the listed slots were used (after every
    // lane's last table read: the shuffles above converge the warp but do not
    // order shared memory, __syncwarp does)
    __syncwarp();
    for (int k = lane; k < nuniq; k += 32) tab[list[k]] = make_int4(-1, 0, 0, 0x7fffffff);
    __syncwarp();
    if (lane == 0) {
        double *pt = a.part + 3 * (size_t)i;
        if (PASS == 1) {
            pt[0] = accS;
            pt[1] = pf;
            pt[2] = pb;
        } else {
            const double dS = pt[0] + accS;
            const double pft = pt[1] + pf;
            const double H = (kout + kin == 0) ? 1.0 : pt[2] / pft;
            const double p = exp(-a.beta * dS) * H;
            const uint32_t itr = a.itr_ptr ? __ldg(a.itr_ptr) : a.itr;
            const uint4 w = draws(a.seed, (uint32_t)v, 0u, itr, a.outer, 1u);
            if (a.dS) a.dS[i] = dS;
            if (a.H) a.H[i] = H;
            if (a.acc) a.acc[i] = ((double)w.w + 0.5) * (1.0 / 4294967296.0) <= p ? 1 : 0;
        }
    }
}

// (a2), one G-thread group (64: a quarter CTA, 256: a CTA) per big vertex:
// every unique block owned by its first adjacency position; threads sum their
// owned terms in position order.
// phase A of a group vertex: its neighbour-block table, built by group
// threads [t0, G) (t0 = 32 when warp 0 of the group is drawing the proposal)
template <int G, bool WEIGHTED>
GSAP_DEV void group_table(const MoveArgs &a, int v, int ro, int nout, int ci, int deg, int4 *tab, int log2cap,
                          int t0) {
    const bool has_self = __ldg(a.selfw + v) > 0;
    for (int j = (int)(threadIdx.x % G) - t0; j < deg; j += G - t0) {
        if (j < 0) break;
        const bool out = j < nout;
        if (nb_self(a, v, has_self, ro, nout, ci, j)) continue;   // the self-loop is carried by selfw
        const int t = nb_block(a, ro, nout, ci, j);
        const int wt = WEIGHTED ? (out ? __ldg(a.wgt + ro + j) : __ldg(a.cscwgt + ci + j - nout)) : 1;
        const int sl = tab_insert(tab, log2cap, t);
        atomicAdd(out ? &tab[sl].y : &tab[sl].z, wt);
        atomicMin(&tab[sl].w, j);
    }
}

// phase B of a group vertex (table complete): every unique block owned by its
// first adjacency position; threads sum their owned terms in position order.
template <int G, bool WEIGHTED>
GSAP_DEV void eval_move_group(const MoveArgs &a, int v, int r, int s, uint4 w, int ro, int nout, int ci, int deg,
                              int4 *tab, int log2cap, double *sh, double &dS_out, double &H_out, bool &acc_out) {
    const int gt = threadIdx.x % G;
    MoveCtx q;
    move_ctx(a, v, r, s, tab, log2cap, q);
    double accS = 0.0, pf = 0.0, pb = 0.0;
    const bool has_self = q.l > 0;
    for (int j = gt; j < deg; j += G) {
        if (nb_self(a, v, has_self, ro, nout, ci, j)) continue;
        const int4 e = tab[tab_find(tab, log2cap, nb_block(a, ro, nout, ci, j))];
        if (e.w != j) continue;
        t_terms(a, q, e.x, e.y, e.z, accS, pf, pb);
    }
    if (gt < 10) core_term(a, q, gt, accS, pf, pb);
    group_sum3<G>(accS, pf, pb, sh);
    mh_decide(a, q, w, accS, pf, pb, dS_out, H_out, acc_out);
}

// the proposal of a group vertex, by one whole warp (R:O.4; same integer
// result as propose_move_thread): the weighted neighbour by a warp prefix
// scan of the weights (unweighted: direct index), the walk over row /
// column u by the 32-ary warp search
template <bool WEIGHTED>
GSAP_DEV int propose_vertex_warp(const MoveArgs &a, int v, uint4 w, int ro, int nout, int ci, int deg) {
    const uint32_t B = (uint32_t)a.B;
    const uint32_t K = (uint32_t)(__ldg(a.kout + v) + __ldg(a.kin + v));
    if (K == 0) return (int)pick(w.z, B);
    const uint32_t p = pick(w.x, K);
    int n;   // the chosen adjacency entry (out entries, then in entries)
    if (!WEIGHTED) {
        n = (int)p;
    } else {
        const int lane = threadIdx.x & 31;
        long long base = 0;
        n = -1;
        for (int j0 = 0; j0 < deg && n < 0; j0 += 32) {
            const int j = j0 + lane;
            const int wt = j < deg ? (j < nout ? __ldg(a.wgt + ro + j) : __ldg(a.cscwgt + ci + j - nout)) : 0;
            int incl = wt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(FULL, incl, o);
                if (lane >= o) incl += t;
            }
            const unsigned bal = __ballot_sync(FULL, j < deg && base + incl > (long long)p);
            if (bal) n = j0 + __ffs(bal) - 1;
            base += __shfl_sync(FULL, incl, 31);
        }
    }
    const int u = nb_block(a, ro, nout, ci, n);
    const uint32_t du = (uint32_t)bm_deg(a.m, u);
    if (coin_random(w.y, B, du)) return (int)pick(w.z, B);
    if (a.m.mt) return __ldg(a.m.mt + u);   // N4
    return bm_walk_warp(a.m, u, (long long)pick(w.z, du));
}

template <int G>
GSAP_DEV void tab_clear(int4 *tab, int slots, int gt) {
    for (int i = gt; i < slots; i += G) tab[i] = make_int4(-1, 0, 0, 0x7fffffff);
}

// outputs of vertex v (index i = v - first) given its proposal s
template <int G, bool WEIGHTED>
GSAP_DEV void do_vertex(const MoveArgs &a, int v, int4 *tab, int log2cap, int *list, double *sh) {
    const int i = v - a.first;
    const uint32_t itr = a.itr_ptr ? __ldg(a.itr_ptr) : a.itr;
    const uint4 w = draws(a.seed, (uint32_t)v, 0u, itr, a.outer, 1u);
    const int gt = threadIdx.x % G;
    const int ro = __ldg(a.rowptr + v), nout = __ldg(a.rowptr + v + 1) - ro;
    const int ci = __ldg(a.cscptr + v), nin = __ldg(a.cscptr + v + 1) - ci;
    const int deg = nout + nin;
    const int r = __ldg(a.b + v);
    // phase A beside the proposal: warp 0 of the group draws s (fused mode),
    // the other threads build the neighbour-block table (it does not depend on s)
    int *sp = reinterpret_cast<int *>(sh + 3 * (G / 32));
    if (a.propose && gt < 32) {
        const int s0 = propose_vertex_warp<WEIGHTED>(a, v, w, ro, nout, ci, deg);
        if (gt == 0) {
            *sp = s0;
            a.s_out[i] = s0;
        }
    } else {
        group_table<G, WEIGHTED>(a, v, ro, nout, ci, deg, tab, log2cap, a.propose ? 32 : 0);
    }
    gsync<G>();
    const int s = a.propose ? *sp : a.s_in[i];
    double dS = 0.0, H = 1.0;
    bool acc = false;
    if (s != r) eval_move_group<G, WEIGHTED>(a, v, r, s, w, ro, nout, ci, deg, tab, log2cap, sh, dS, H, acc);
    if ((threadIdx.x & (G - 1)) == 0) {
        if (a.dS) a.dS[i] = dS;
        if (a.H) a.H[i] = H;
        if (a.acc) a.acc[i] = acc ? 1 : 0;
    }
}

template <bool WEIGHTED>
__global__ void __launch_bounds__(256) k_propose(MoveArgs a) {
    const uint32_t itr = a.itr_ptr ? __ldg(a.itr_ptr) : a.itr;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < a.count; i += gridDim.x * blockDim.x) {
        const int v = a.first + i;
        const uint4 w = draws(a.seed, (uint32_t)v, 0u, itr, a.outer, 1u);
        a.s_out[i] = propose_move_thread<WEIGHTED>(a, v, w);
    }
}

// One launch, two roles: CTAs [0, nbig_ctas) take the vertices of a.list
// (whose neighbour-block count can exceed 128) one CTA per vertex; the other
// CTAs take every other vertex of [first, first + count) one warp per vertex.
// The shared memory is the 8 warp tables, or one CTA table over the same bytes.
template <bool WEIGHTED>
#ifndef GSAP_GROUPS_MINB
#define GSAP_GROUPS_MINB 2
#endif
__global__ void __launch_bounds__(MOVE_WARPS * 32, GSAP_GROUPS_MINB) k_move_groups(MoveArgs a) {
    __shared__ int4 tabs[CTA_SMEM_SLOTS];
    __shared__ double sh[3 * MOVE_WARPS + 8];   // group sums + the broadcast proposal
    if ((int)blockIdx.x < a.nmid_ctas) {
        // MID_PER_CTA groups of MID_G threads per CTA, one mid vertex each
        const int gid = threadIdx.x / MID_G, gt = threadIdx.x % MID_G;
        int4 *tab = tabs + gid * MID_TAB;
        for (int li = blockIdx.x * MID_PER_CTA + gid; li < a.mlist_count; li += a.nmid_ctas * MID_PER_CTA) {
            tab_clear<MID_G>(tab, MID_TAB, gt);
            gsync<MID_G>();
            do_vertex<MID_G, WEIGHTED>(a, a.mlist[li], tab, MID_TAB_LOG2, nullptr,
                                       sh + gid * ((3 * MOVE_WARPS + 8) / MID_PER_CTA));
            gsync<MID_G>();
        }
        return;
    }
    if ((int)blockIdx.x < a.nmid_ctas + a.nbig_ctas) {
        for (int li = blockIdx.x - a.nmid_ctas; li < a.list_count; li += a.nbig_ctas) {
            tab_clear<CTA_THREADS>(tabs, 1 << a.big_log2, threadIdx.x);
            __syncthreads();
            do_vertex<CTA_THREADS, WEIGHTED>(a, a.list[li], tabs, a.big_log2, nullptr, sh);
            __syncthreads();
        }
        return;
    }
    if ((int)blockIdx.x < a.nmid_ctas + a.nbig_ctas + a.nhuge_ctas) {
        const int hb = blockIdx.x - a.nmid_ctas - a.nbig_ctas;
        int4 *tab = a.gtab ? a.gtab + ((size_t)hb << a.gtab_log2) : tabs;
        for (int li = hb; li < a.hlist_count; li += a.nhuge_ctas) {
            tab_clear<CTA_THREADS>(tab, 1 << a.gtab_log2, threadIdx.x);
            __syncthreads();
            do_vertex<CTA_THREADS, WEIGHTED>(a, a.hlist[li], tab, a.gtab_log2, nullptr, sh);
            __syncthreads();
        }
        }
}

// (a1 + a2) warp role: every vertex of [first, first + count) that is not in
// a group list, one warp per vertex (launched beside k_move_groups)
template <bool WEIGHTED, bool DENSE>
__global__ void __launch_bounds__(MOVE_WARPS * 32, GSAP_MOVE_MINB) k_move(MoveArgs a) {
    extern __shared__ int4 move_smem[];   // MOVE_SMEM bytes
    int4 *tabs = move_smem;                                         // MOVE_WARPS * WARP_TAB
    int *lists = reinterpret_cast<int *>(tabs + MOVE_WARPS * WARP_TAB);   // MOVE_WARPS * WARP_TAB / 2
    const int wl = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int4 *tab = tabs + wl * WARP_TAB;
    int *list = lists + wl * (WARP_TAB / 2);
    tab_clear<32>(tab, WARP_TAB, lane);
    __syncwarp();
    const int nwarps = gridDim.x * MOVE_WARPS;
    const bool skip_big = a.B > BIG_THR;
    for (int i = blockIdx.x * MOVE_WARPS + wl; i < a.count; i += nwarps) {
        const int v = a.first + i;
        // adjacency entries bound the number of unique neighbour blocks
        if (skip_big &&
            (__ldg(a.rowptr + v + 1) - __ldg(a.rowptr + v)) + (__ldg(a.cscptr + v + 1) - __ldg(a.cscptr + v)) > BIG_THR)
            continue;
        move_vertex_warp<WEIGHTED, DENSE>(a, i, tab, list);
    }
}

// sorted two-pass mode: warp w takes batch index perm[w] (grid-stride), so
// consecutive warps search the same key's two lines (hits in L1 / L2)
#ifndef GSAP_HALF_MINB
#define GSAP_HALF_MINB 4
#endif
template <bool WEIGHTED, int PASS>
__global__ void __launch_bounds__(MOVE_WARPS * 32, GSAP_HALF_MINB) k_move_half(MoveArgs a) {
    extern __shared__ int4 move_smem[];   // MOVE_SMEM bytes
    int4 *tabs = move_smem;
    int *lists = reinterpret_cast<int *>(tabs + MOVE_WARPS * WARP_TAB);
    const int wl = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int4 *tab = tabs + wl * WARP_TAB;
    int *list = lists + wl * (WARP_TAB / 2);
    tab_clear<32>(tab, WARP_TAB, lane);
    __syncwarp();
    const int nwarps = gridDim.x * MOVE_WARPS;
    for (int w = blockIdx.x * MOVE_WARPS + wl; w < a.count; w += nwarps) {
        const int i = __ldg(a.perm + w);
        const int v = a.first + i;
        if ((__ldg(a.rowptr + v + 1) - __ldg(a.rowptr + v)) + (__ldg(a.cscptr + v + 1) - __ldg(a.cscptr + v)) > BIG_THR)
            continue;
        move_vertex_half<WEIGHTED, PASS>(a, i, tab, list);
    }
}

// counting sort of the batch by r = b[v] (keys [0, B)) and by s (keys [B, 2B)):
// counts, then (after an exclusive scan of both) the scatter into perm[0, 2 count)
__global__ void __launch_bounds__(256) k_sort_count(int first, int count, const int *__restrict__ b,
                                                    const int *__restrict__ s, int B, int *__restrict__ cnt) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < count; i += gridDim.x * blockDim.x) {
        atomicAdd(cnt + __ldg(b + first + i), 1);
        atomicAdd(cnt + B + __ldg(s + i), 1);
    }
}

__global__ void __launch_bounds__(256) k_sort_scatter(int first, int count, const int *__restrict__ b,
                                                      const int *__restrict__ s, int B, int *__restrict__ off,
                                                      int *__restrict__ perm) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < count; i += gridDim.x * blockDim.x) {
        perm[atomicAdd(off + __ldg(b + first + i), 1)] = i;
        perm[atomicAdd(off + B + __ldg(s + i), 1)] = i;   // offsets of the s keys start at count
    }
}

// ------------------------------------------------------------------ host --
static int log2_ceil(long long x) {
    int l = 0;
    while ((1LL << l) < x) ++l;
    return l;
}

void launch_move(Ctx &c, MoveMode mode, uint32_t outer, uint32_t itr, int first, int count, int *s, double *dS,
                 double *H, unsigned char *acc, const unsigned *d_itr) {
    if (count <= 0) return;
    nb_join(c);   // the move kernels read the neighbour-block cache
    cudaEvent_t ev = nullptr;
    kc_begin(c, c.k_move, &ev);
    MoveArgs a;
    a.B = c.B;
    a.seed = c.prm.seed;
    a.outer = outer;
    a.itr = itr;
    a.itr_ptr = d_itr;
    a.beta = c.prm.beta;
    a.rowptr = c.rowptr; a.col = c.col; a.wgt = c.wgt;
    a.cscptr = c.cscptr; a.cscsrc = c.cscsrc; a.cscwgt = c.cscwgt;
    a.kout = c.kout; a.kin = c.kin; a.selfw = c.selfw; a.b = c.b;
    a.nbo = c.nbo; a.nbi = c.nbi;
    a.m = c.bm();
    a.first = first;
    a.count = count;
    a.list = nullptr;
    a.list_count = 0;
    a.s_in = s;
    a.s_out = s;
    a.dS = dS; a.H = H; a.acc = acc;
    a.gtab = nullptr;
    a.gtab_log2 = 0;
    a.perm = nullptr;
    a.part = nullptr;
    a.propose = mode == MOVE_FUSED ? 1 : 0;
    // sorted two-pass evaluation of a fused batch (large sparse blockmodels)
    // decided per MOVE batch (c.batch_count), not per slice: the same mode for any number of GPUs
    const int bc = c.batch_count > 0 ? c.batch_count : count;
    const bool sorted = mode == MOVE_FUSED && a.m.dense == nullptr && c.B > BIG_THR &&
                        (c.prm.move_sorted == 2 || (c.prm.move_sorted == 1 && (long long)c.E > GSAP_COOP_MAX_E &&
                                                    bc >= (1 << 16)));
    if (mode == MOVE_PROPOSE || sorted) {   // (a1) alone: thread per vertex
        const int pg = (int)std::min<long long>(((long long)count + 63) / 64, 148LL * 64);
        if (c.weighted) k_propose<true><<<pg, 64, 0, c.stream>>>(a);
        else k_propose<false><<<pg, 64, 0, c.stream>>>(a);
        ++c.launches;
        GSAP_CHECK_LAUNCH();
        if (!sorted) {
            kc_end(c, c.k_move, ev, 0.0);
            return;
        }
        // group the batch by r and by s (counting sort; the order inside a
        // group is irrelevant: every vertex reads the same snapshot)
        const int B = c.B;
        Launcher L{c.stream, &c.launches};
        GSAP_CUDA(cudaMemsetAsync(c.mv_cnt, 0, sizeof(int) * 2 * (size_t)B, c.stream));
        const int sg = (int)std::min<long long>(((long long)count + 255) / 256, 148LL * 16);
        k_sort_count<<<sg, 256, 0, c.stream>>>(first, count, c.b, s, B, c.mv_cnt);
        device_scan<int>(c.mv_cnt, c.mv_cnt, nullptr, 2 * B, false, c.mv_scan_tmp, nullptr, L);
        k_sort_scatter<<<sg, 256, 0, c.stream>>>(first, count, c.b, s, B, c.mv_cnt, c.mv_perm);
        c.launches += 2;
        GSAP_CHECK_LAUNCH();
        a.propose = 0;          // groups and both passes read the proposals s
        a.part = c.mv_part;
    }
    a.nbig_ctas = 0;
    a.nhuge_ctas = 0;
    a.nmid_ctas = 0;
    a.mlist = nullptr;
    a.mlist_count = 0;
    a.hlist = nullptr;
    a.hlist_count = 0;
    a.big_log2 = 5;
    if (c.B > BIG_THR) {
        // the big (128 < k <= 1024) and huge (k > 1024) vertices inside [first, first + count)
        auto range = [&](const std::vector<int> &h, int &n, int &kmax) {
            const auto lo = std::lower_bound(h.begin(), h.end(), first);
            const auto hi = std::lower_bound(h.begin(), h.end(), first + count);
            n = (int)(hi - lo);
            kmax = 0;
            for (auto it = lo; it != hi; ++it) {
                const int v = *it;
                kmax = std::max(kmax, (c.h_rowptr[v + 1] - c.h_rowptr[v]) + (c.h_cscptr[v + 1] - c.h_cscptr[v]));
            }
            return (int)(lo - h.begin());
        };
        int nmid = 0, kmid = 0, nbig = 0, kbig = 0, nhuge = 0, khuge = 0;
        const int omid = range(c.h_mid, nmid, kmid);
        int obig = range(c.h_big, nbig, kbig);
#ifndef GSAP_GROUPS_LATENCY
#define GSAP_GROUPS_LATENCY 0
#endif
        // latency mode (build flag): few group vertices in the batch -- the
        // 129..256-entry vertices get a whole CTA each like the bigger ones
        if (GSAP_GROUPS_LATENCY && nmid > 0 && nmid + nbig <= 2 * 148 * GSAP_GROUPS_MINB) {
            int n2 = 0, k2 = 0;
            const int o2 = range(c.h_midbig, n2, k2);
            a.list = c.midbig + o2;
            a.list_count = n2;
            a.big_log2 = std::max(log2_ceil(2LL * std::min(k2, c.B)), 5);
            a.nbig_ctas = std::min(n2, c.test_grid > 0 ? c.test_grid : 148 * 16);
            nmid = 0;
            nbig = 0;
        }
        if (nmid > 0) {
            a.mlist = c.mid + omid;
            a.mlist_count = nmid;
            a.nmid_ctas = std::min((nmid + MID_PER_CTA - 1) / MID_PER_CTA, c.test_grid > 0 ? c.test_grid : 148 * 16);
        }
        const int ohuge = range(c.h_huge, nhuge, khuge);
        if (nbig > 0) {
            a.list = c.big + obig;
            a.list_count = nbig;
            a.big_log2 = std::max(log2_ceil(2LL * std::min(kbig, c.B)), 5);   // <= 11: shared
            a.nbig_ctas = std::min(nbig, c.test_grid > 0 ? c.test_grid : 148 * 16);
        }
        if (nhuge > 0) {
            a.hlist = c.huge + ohuge;
            a.hlist_count = nhuge;
            a.gtab_log2 = std::max(log2_ceil(2LL * std::min(khuge, c.B)), 5);
            if ((1 << a.gtab_log2) > CTA_SMEM_SLOTS) {
                a.nhuge_ctas = (int)std::min<long long>(nhuge, (long long)(c.big_table_slots >> a.gtab_log2));
                if (a.nhuge_ctas < 1) throw Error{GSAP_ENOMEM, "huge-vertex table too small"};
                a.gtab = reinterpret_cast<int4 *>(c.big_tables);
            } else {
                a.nhuge_ctas = std::min(nhuge, c.test_grid > 0 ? c.test_grid : 148 * 16);
            }
        }
    }
    const long long need = ((long long)count + MOVE_WARPS - 1) / MOVE_WARPS;
    // c.test_grid (tests only, GSAP_TEST_GRID): a few CTAs striding over
    // everything -- the results must not depend on the launch shape
    const int grid = (int)std::max<long long>(1, std::min<long long>(need, c.test_grid > 0 ? c.test_grid : 148LL * 8));
    const int ggrid = a.nmid_ctas + a.nbig_ctas + a.nhuge_ctas;
    if (ggrid > 0) {   // the group roles run beside the warp role (fork / join on the side stream)
        GSAP_CUDA(cudaEventRecord(c.ev_fork, c.stream));
        GSAP_CUDA(cudaStreamWaitEvent(c.side, c.ev_fork, 0));
        cudaEvent_t rg = role_begin(c, c.k_groups, c.side);
        if (c.weighted) k_move_groups<true><<<ggrid, MOVE_WARPS * 32, 0, c.side>>>(a);
        else k_move_groups<false><<<ggrid, MOVE_WARPS * 32, 0, c.side>>>(a);
        role_end(c, c.k_groups, rg, c.side);
        ++c.launches;
        GSAP_CHECK_LAUNCH();
        GSAP_CUDA(cudaEventRecord(c.ev_join, c.side));
    }
    per_device((const void *)k_move<false, false>, [] {
        const int sm = (int)MOVE_SMEM;
        GSAP_CUDA(cudaFuncSetAttribute(k_move<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
        GSAP_CUDA(cudaFuncSetAttribute(k_move<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
        GSAP_CUDA(cudaFuncSetAttribute(k_move<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
        GSAP_CUDA(cudaFuncSetAttribute(k_move<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
        return 1;
    });
    const bool dense = a.m.dense != nullptr;
    cudaEvent_t rw = role_begin(c, c.k_warps, c.stream);
    if (sorted) {
        per_device((const void *)k_move_half<false, 1>, [] {
            const int sm = (int)MOVE_SMEM;
            GSAP_CUDA(cudaFuncSetAttribute(k_move_half<true, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
            GSAP_CUDA(cudaFuncSetAttribute(k_move_half<true, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
            GSAP_CUDA(cudaFuncSetAttribute(k_move_half<false, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
            GSAP_CUDA(cudaFuncSetAttribute(k_move_half<false, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm));
            return 1;
        });
        MoveArgs a1 = a, a2 = a;
        a1.perm = c.mv_perm;            // grouped by r
        a2.perm = c.mv_perm + count;    // grouped by s
        if (c.weighted) {
            k_move_half<true, 1><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a1);
            k_move_half<true, 2><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a2);
        } else {
            k_move_half<false, 1><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a1);
            k_move_half<false, 2><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a2);
        }
        c.launches += 2;
    } else if (c.weighted) {
        if (dense) k_move<true, true><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a);
        else k_move<true, false><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a);
        ++c.launches;
    } else {
        if (dense) k_move<false, true><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a);
        else k_move<false, false><<<grid, MOVE_WARPS * 32, MOVE_SMEM, c.stream>>>(a);
        ++c.launches;
    }
    GSAP_CHECK_LAUNCH();
    role_end(c, c.k_warps, rw, c.stream);
    if (ggrid > 0) GSAP_CUDA(cudaStreamWaitEvent(c.stream, c.ev_join, 0));
    // algorithmic bytes: the adjacency ids (+
    // weights), 2 x 16 B of row / column pointers and 13 B of per-vertex
    // state and outputs (b[v], s, dS, acc) per vertex
    const long long adj = (long long)(c.h_rowptr[first + count] - c.h_rowptr[first]) +
                          (c.h_cscptr[first + count] - c.h_cscptr[first]);
    const double bytes = (c.weighted ? 8.0 : 4.0) * adj + 45.0 * count;
    kc_end(c, c.k_move, ev, bytes);
}

// ---------------------------------------------------------------- apply --
constexpr int APPLY_CHUNK = 1024;

// N2 (incremental blockmodel update, P:250-255 3.4): when log.oldb is set,
// every applied move records the vertex's old block (oldb[v]) and appends v
// to log.moved (warp-aggregated atomics, order irrelevant: the update is
// integer additions)
struct MoveLog {
    int *oldb, *moved, *moved_cnt, *movedb;
};

GSAP_DEV void log_move(const MoveLog &lg, bool mv, int v, int old, int nw) {
    const unsigned m = __ballot_sync(FULL, mv);   // warp-uniform call
    if (!m) return;
    const int lane = threadIdx.x & 31, leader = __ffs(m) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(lg.moved_cnt, __popc(m));
    base = __shfl_sync(FULL, base, leader);
    if (mv) {
        lg.oldb[v] = old;
        const int k = base + __popc(m & ((1u << lane) - 1u));
        lg.moved[k] = v;
        lg.movedb[k] = nw;
    }
}

// n_eval (nullable): += the proposals with s != b[v] (the moves that were
// evaluated, R:Z13) -- counted before b is written
__global__ void __launch_bounds__(APPLY_CHUNK) k_apply(int first, int count, const int *__restrict__ s,
                                               const unsigned char *__restrict__ acc,
                                               const double *__restrict__ dS, int *__restrict__ b,
                                               double *__restrict__ partials, int *__restrict__ nacc,
                                               unsigned long long *__restrict__ n_eval, MoveLog lg) {
    __shared__ double sh[APPLY_CHUNK / 32];
    const int base = blockIdx.x * APPLY_CHUNK;
    double sum = 0.0;
    int na = 0, ne = 0;
    {   // one entry of the chunk per thread
        const int k = threadIdx.x;
        const int i = base + k;
        if (i < count && n_eval) ne += s[i] != b[first + i];
        if (lg.oldb) {
            const bool mv = i < count && acc[i];
            log_move(lg, mv, first + i, mv ? b[first + i] : 0, mv ? s[i] : 0);
        }
        if (i < count && acc[i]) {
            if (b) b[first + i] = s[i];
            sum += dS ? dS[i] : 0.0;
            ++na;
        }
    }
    na = warp_sum(na);
    if (nacc && (threadIdx.x & 31) == 0 && na) atomicAdd(nacc, na);
    if (n_eval) {
        ne = warp_sum(ne);
        if ((threadIdx.x & 31) == 0 && ne) atomicAdd(n_eval, (unsigned long long)ne);
    }
    sum = warp_sum(sum);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = sum;
    __syncthreads();
    if (threadIdx.x == 0 && partials) {
        double t = 0.0;
        for (int w = 0; w < APPLY_CHUNK / 32; ++w) t += sh[w];
        partials[blockIdx.x] = t;
    }
}

// out (+)= sum of partials[0, n) in a fixed order
__global__ void __launch_bounds__(256) k_sum_partials(const double *__restrict__ partials, int n,
                                                      double *out, int accumulate) {
    __shared__ double sh[8];
    double v = 0.0;
    for (int i = threadIdx.x; i < n; i += 256) v += partials[i];
    v = warp_sum(v);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < 8; ++w) t += sh[w];
        *out = accumulate ? *out + t : t;
    }
}

// k_apply + the ordered sum of its partials in one launch: the last CTA to
// finish (arrival counter, reset by that CTA) adds partials[0, nb) in index
// order to *dsum -- the same fixed-order sum as k_sum_partials
__global__ void __launch_bounds__(APPLY_CHUNK) k_apply_sum(int first, int count, const int *__restrict__ s,
                                                   const unsigned char *__restrict__ acc,
                                                   const double *__restrict__ dS, int *__restrict__ b,
                                                   double *__restrict__ partials, int *__restrict__ nacc,
                                                   unsigned *__restrict__ arrivals, double *__restrict__ dsum,
                                                   unsigned long long *__restrict__ n_eval, MoveLog lg) {
    __shared__ double sh[APPLY_CHUNK / 32];
    __shared__ bool last;
    const int base = blockIdx.x * APPLY_CHUNK;
    double sum = 0.0;
    int na = 0, ne = 0;
    {   // one entry of the chunk per thread
        const int k = threadIdx.x;
        const int i = base + k;
        if (i < count && n_eval) ne += s[i] != b[first + i];
        if (lg.oldb) {
            const bool mv = i < count && acc[i];
            log_move(lg, mv, first + i, mv ? b[first + i] : 0, mv ? s[i] : 0);
        }
        if (i < count && acc[i]) {
            b[first + i] = s[i];
            sum += dS ? dS[i] : 0.0;
            ++na;
        }
    }
    na = warp_sum(na);
    if (nacc && (threadIdx.x & 31) == 0 && na) atomicAdd(nacc, na);
    if (n_eval) {
        ne = warp_sum(ne);
        if ((threadIdx.x & 31) == 0 && ne) atomicAdd(n_eval, (unsigned long long)ne);
    }
    sum = warp_sum(sum);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = sum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < APPLY_CHUNK / 32; ++w) t += sh[w];
        partials[blockIdx.x] = t;
        __threadfence();
        last = atomicAdd(arrivals, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    double v = 0.0;
    // the order of k_sum_partials: 256 strided lanes, warp trees, 8 warp sums
    if (threadIdx.x < 256)
        for (int i = threadIdx.x; i < (int)gridDim.x; i += 256) v += *((volatile double *)(partials + i));
    v = warp_sum(v);
    if ((threadIdx.x & 31) == 0 && threadIdx.x < 256) sh[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < 8; ++w) t += sh[w];
        *dsum += t;
        *arrivals = 0u;
    }
}

// argument validation of device inputs (gsap_set_partition, gsap_apply_moves,
// gsap_select_merges): *bad = 1 if some x[i] (with mask[i] != 0, if a mask is
// given) lies outside [0, B), or equals i when not_self
__global__ void k_check_ids(int n, const int *__restrict__ x, const unsigned char *__restrict__ mask, int B,
                            int not_self, int *__restrict__ bad) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        if (mask && !mask[i]) continue;
        const int v = x[i];
        if (v < 0 || v >= B || (not_self && v == i)) *bad = 1;
    }
}

bool device_ids_ok(Ctx &c, int n, const int *x, const unsigned char *mask, int B, bool not_self) {
    if (n <= 0) return true;
    GSAP_CUDA(cudaMemsetAsync(c.scal_i + 6, 0, sizeof(int), c.stream));
    const int g = (int)std::min<long long>(((long long)n + 255) / 256, 148LL * 8);
    k_check_ids<<<g, 256, 0, c.stream>>>(n, x, mask, B, not_self ? 1 : 0, c.scal_i + 6);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
    GSAP_CUDA(cudaMemcpyAsync(c.h_int + 6, c.scal_i + 6, sizeof(int), cudaMemcpyDeviceToHost, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    return c.h_int[6] == 0;
}

// the neighbour-block cache after an apply (internal.h Ctx::nbo): every moved
// vertex v (the apply's move log) rewrites its own entries in its neighbours'
// lists -- the in-edges u -> v hold v's block at CSR position csc2csr[q] (q in
// v's CSC range), the out-edges v -> w at CSC position csr2csc[p] (p in v's
// CSR range); each position belongs to one edge, so the writes never collide.
// One warp per moved vertex.
__global__ void __launch_bounds__(256) k_nb_update(const int *__restrict__ moved, const int *__restrict__ moved_cnt,
                                                   const int *__restrict__ movedb, const int *__restrict__ rowptr,
                                                   const int *__restrict__ cscptr, const int *__restrict__ csc2csr,
                                                   const int *__restrict__ csr2csc, int *__restrict__ nbo,
                                                   int *__restrict__ nbi) {
    const int n = *moved_cnt, lane = threadIdx.x & 31;
    for (int k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < n; k += (gridDim.x * blockDim.x) >> 5) {
        const int v = moved[k];
        const int x = movedb[k];   // the new block, from the log (not b: the update may run beside later writes of b)
        const int q1 = __ldg(cscptr + v + 1), p1 = __ldg(rowptr + v + 1);
        for (int q = __ldg(cscptr + v) + lane; q < q1; q += 32) nbo[__ldg(csc2csr + q)] = x;
        for (int p = __ldg(rowptr + v) + lane; p < p1; p += 32) nbi[__ldg(csr2csc + p)] = x;
    }
}

static void launch_nb_update(Ctx &c, int count);

void nb_flush(Ctx &c) {
    if (!c.nb_deferred) return;
    c.nb_deferred = false;
    const int g = 148 * 8;
    k_nb_update<<<g, 256, 0, c.stream>>>(c.moved, c.moved_cnt, c.movedb, c.rowptr, c.cscptr, c.csc2csr, c.csr2csc,
                                         c.nbo, c.nbi);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
}

void nb_join(Ctx &c, bool flush) {
    if (flush) nb_flush(c);
    if (!c.nb_pending) return;
    GSAP_CUDA(cudaStreamWaitEvent(c.stream, c.ev_nb, 0));
    c.nb_pending = false;
}

// the cache update after an apply.  In the dense regime the rebuild that
// follows reads b and M only, so the update runs on the side stream beside
// it and the next reader of nbo / nbi joins it (nb_join); elsewhere in order.
static void launch_nb_update(Ctx &c, int count) {
    if (!c.nbo || c.nb_stale) return;   // a stale cache is refreshed in full by the next rebuild
    static const bool in_order = getenv("GSAP_NB_INORDER") != nullptr;   // A/B switch
    static const bool no_defer = getenv("GSAP_NB_NODEFER") != nullptr;   // A/B switch
    const bool side = !in_order && c.dense_mode && dense_ok(c, c.B) && c.nranks == 1;
    nb_join(c);
    if (!no_defer && !dense_ok(c, c.B) && c.coop_ok && c.E > 0) {
        c.nb_deferred = true;   // done by the persistent sparse rebuild's first phase
        return;
    }
    cudaStream_t st = c.stream;
    if (side) {
        GSAP_CUDA(cudaEventRecord(c.ev_apply, c.stream));
        GSAP_CUDA(cudaStreamWaitEvent(c.side, c.ev_apply, 0));
        st = c.side;
    }
    const int g = (int)std::min<long long>(((long long)count + 7) / 8, 148LL * 8);
    k_nb_update<<<g, 256, 0, st>>>(c.moved, c.moved_cnt, c.movedb, c.rowptr, c.cscptr, c.csc2csr, c.csr2csc,
                                   c.nbo, c.nbi);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
    if (side) {
        GSAP_CUDA(cudaEventRecord(c.ev_nb, c.side));
        c.nb_pending = true;
    }
}

// the move log of the batch: for the incremental update (N2, when the caller
// announced the batch and the regime keeps dense M) and the neighbour-block cache
static MoveLog move_log(Ctx &c) {
    MoveLog lg{nullptr, nullptr, nullptr, nullptr};
    if (c.delta.pending || c.nbo) {
        GSAP_CUDA(cudaMemsetAsync(c.moved_cnt, 0, sizeof(int), c.stream));
        lg = MoveLog{c.oldb, c.moved, c.moved_cnt, c.movedb};
    }
    return lg;
}

void launch_apply(Ctx &c, int first, int count, const int *s, const unsigned char *acc, const double *dS,
                  double *dsum, int *nacc, unsigned long long *n_eval) {
    if (count <= 0) return;
    const int nb = (count + APPLY_CHUNK - 1) / APPLY_CHUNK;
    const MoveLog lg = move_log(c);
    k_apply_sum<<<nb, APPLY_CHUNK, 0, c.stream>>>(first, count, s, acc, dS, c.b, c.partials, nacc,
                                          reinterpret_cast<unsigned *>(c.scal_i + 4), dsum, n_eval, lg);
    c.launches += 1;
    GSAP_CHECK_LAUNCH();
    launch_nb_update(c, count);
}

void launch_apply_deferred(Ctx &c, int first, int count, const int *s, const unsigned char *acc, const double *dS,
                           double *part, int *nacc, unsigned long long *n_eval) {
    if (count <= 0) return;
    const int nb = (count + APPLY_CHUNK - 1) / APPLY_CHUNK;
    const MoveLog lg = move_log(c);
    k_apply<<<nb, APPLY_CHUNK, 0, c.stream>>>(first, count, s, acc, dS, c.b, part, nacc, n_eval, lg);
    c.launches += 1;
    GSAP_CHECK_LAUNCH();
    launch_nb_update(c, count);
}

// sharded batches: the fixed-chunk sums of accepted dS over [first, first+count)
// (first aligned to APPLY_CHUNK from the batch start) into partials[0, ...)
void launch_partials(Ctx &c, int first, int count, const int *s, const unsigned char *acc, const double *dS,
                     double *partials) {
    if (count <= 0) return;
    const int nb = (count + APPLY_CHUNK - 1) / APPLY_CHUNK;
    k_apply<<<nb, APPLY_CHUNK, 0, c.stream>>>(first, count, s, acc, dS, nullptr, partials, nullptr, nullptr,
                                      MoveLog{nullptr, nullptr, nullptr, nullptr});
    ++c.launches;
    GSAP_CHECK_LAUNCH();
}

// sharded batches: apply all gathered moves, then the ordered sum of n partials
void launch_apply_gathered(Ctx &c, int first, int count, const int *s, const unsigned char *acc,
                           const double *partials, int n, double *dsum, int *nacc, unsigned long long *n_eval) {
    if (count <= 0) return;
    const int nb = (count + APPLY_CHUNK - 1) / APPLY_CHUNK;
    const MoveLog lg = move_log(c);
    k_apply<<<nb, APPLY_CHUNK, 0, c.stream>>>(first, count, s, acc, nullptr, c.b, nullptr, nacc, n_eval, lg);
    k_sum_partials<<<1, 256, 0, c.stream>>>(partials, n, dsum, 1);
    c.launches += 2;
    GSAP_CHECK_LAUNCH();
    launch_nb_update(c, count);
}

}  // namespace gsap
