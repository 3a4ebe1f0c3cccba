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

#include "internal.h"

namespace gsap {

constexpr int WARP_TAB = 256;          // slots per warp table (<= 128 keys)
constexpr int WARP_TAB_LOG2 = 8;
constexpr int BIG_THR = 128;           // warp path iff min(k_v, B) <= BIG_THR
constexpr int MOVE_WARPS = 8;          // warps per CTA, warp kernel
constexpr int CTA_THREADS = 256;       // big-vertex role: one CTA per vertex
constexpr int CTA_SMEM_SLOTS = MOVE_WARPS * WARP_TAB;   // big-vertex shared table (<= 1024 keys)
constexpr int BIG_CTAS_MAX = 296;      // CTAs of the big-vertex role (grid-stride)

struct MoveArgs {
    int B;
    uint64_t seed;
    uint32_t outer, itr;
    const unsigned *itr_ptr;        // if set, the iteration is read from the device
    double beta;
    const int *__restrict__ rowptr, *__restrict__ col, *__restrict__ wgt;
    const int *__restrict__ cscptr, *__restrict__ cscsrc, *__restrict__ cscwgt;
    const int *__restrict__ kout, *__restrict__ kin, *__restrict__ selfw, *__restrict__ b;
    BM m;
    int first, count;
    const int *__restrict__ list;   // big-vertex kernel: sorted vertex ids
    int list_count;
    const int *s_in;                // MOVE_DELTA
    int *s_out;
    double *dS, *H;
    unsigned char *acc;
    int4 *gtab;                     // global tables (big-vertex role), per CTA, or nullptr
    int gtab_log2;
    int nbig_ctas;                  // CTAs [0, nbig_ctas) take the big-vertex role
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

// weighted pick over ids[lo, lo+len) by weights wts; p is reduced by the list
// total when the pick falls beyond it (returns -1).  Whole warp.
GSAP_DEV int warp_pick(const int *__restrict__ ids, const int *__restrict__ wts, int lo, int len, long long &p) {
    const int lane = threadIdx.x & 31;
    long long carry = 0;
    for (int base = 0; base < len; base += 32) {
        const int j = base + lane;
        const int wv = j < len ? __ldg(wts + lo + j) : 0;
        const int id = j < len ? __ldg(ids + lo + j) : -1;
        const int sc = warp_incl_scan(wv);
        const unsigned bal = __ballot_sync(FULL, j < len && carry + sc > p);
        if (bal) return __shfl_sync(FULL, id, __ffs(bal) - 1);
        carry += __shfl_sync(FULL, sc, 31);
    }
    p -= carry;
    return -1;
}

// (a1) MOVE proposal for v (R:O.4).  Whole warp; result warp-uniform.
template <bool WEIGHTED>
GSAP_DEV int propose_move(const MoveArgs &a, int v, uint4 w) {
    const uint32_t B = (uint32_t)a.B;
    const uint32_t K = (uint32_t)(__ldg(a.kout + v) + __ldg(a.kin + v));
    if (K == 0) return (int)pick(w.z, B);
    const int ro = __ldg(a.rowptr + v), nout = __ldg(a.rowptr + v + 1) - ro;
    const int ci = __ldg(a.cscptr + v), nin = __ldg(a.cscptr + v + 1) - ci;
    int n;
    if (!WEIGHTED) {
        const uint32_t p = pick(w.x, K);
        n = (int)p < nout ? __ldg(a.col + ro + p) : __ldg(a.cscsrc + ci + (p - nout));
    } else {
        long long p = pick(w.x, K);
        n = warp_pick(a.col, a.wgt, ro, nout, p);
        if (n < 0) n = warp_pick(a.cscsrc, a.cscwgt, ci, nin, p);
    }
    const int u = __ldg(a.b + n);
    const uint32_t du = (uint32_t)bm_deg(a.m, u);
    if (coin_random(w.y, B, du)) return (int)pick(w.z, B);
    return bm_walk_warp(a.m, u, (long long)pick(w.z, du));
}

// group-wide sums (deterministic fixed trees)
template <int G>
GSAP_DEV double group_sum(double v, double *sh) {
    v = warp_sum(v);
    if (G == 32) return v;
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    __syncthreads();
    if (lane == 0) sh[w] = v;
    __syncthreads();
    double t = 0.0;
#pragma unroll
    for (int i = 0; i < G / 32; ++i) t += sh[i];
    __syncthreads();
    return t;
}

template <int G>
GSAP_DEV void group_sync() {
    if (G == 32) __syncwarp();
    else __syncthreads();
}

// (a2) Delta S + Hastings + MH accept for v: r -> s, r != s, on the table
// `tab` (2^log2cap slots, empty on entry).  gt = thread index in the group.
template <int G, bool WEIGHTED>
GSAP_DEV void eval_move(const MoveArgs &a, int v, int s, uint4 w, int4 *tab, int log2cap, int gt,
                        double *sh, double &dS_out, double &H_out, bool &acc_out) {
    const int B = a.B;
    const int r = __ldg(a.b + v);
    const int ro = __ldg(a.rowptr + v), nout = __ldg(a.rowptr + v + 1) - ro;
    const int ci = __ldg(a.cscptr + v), nin = __ldg(a.cscptr + v + 1) - ci;
    const int deg = nout + nin;
    // phase A: histogram of neighbour blocks
    for (int j = gt; j < deg; j += G) {
        const bool out = j < nout;
        const int nb = out ? __ldg(a.col + ro + j) : __ldg(a.cscsrc + ci + j - nout);
        if (nb == v) continue;   // the self-loop is carried by selfw
        const int t = __ldg(a.b + nb);
        const int wt = WEIGHTED ? (out ? __ldg(a.wgt + ro + j) : __ldg(a.cscwgt + ci + j - nout)) : 1;
        const int sl = tab_insert(tab, log2cap, t);
        atomicAdd(out ? &tab[sl].y : &tab[sl].z, wt);
        atomicMin(&tab[sl].w, j);
    }
    group_sync<G>();
    // 2x2 core (every thread, redundantly: broadcast loads)
    const long long Mrr = bm_at(a.m, r, r), Mrs = bm_at(a.m, r, s);
    const long long Msr = bm_at(a.m, s, r), Mss = bm_at(a.m, s, s);
    const int slr = tab_find(tab, log2cap, r), sls = tab_find(tab, log2cap, s);
    const long long o_r = slr >= 0 ? tab[slr].y : 0, i_r = slr >= 0 ? tab[slr].z : 0;
    const long long o_s = sls >= 0 ? tab[sls].y : 0, i_s = sls >= 0 ? tab[sls].z : 0;
    const long long kout = __ldg(a.kout + v), kin = __ldg(a.kin + v), l = __ldg(a.selfw + v);
    const long long dr = bm_deg(a.m, r), ds = bm_deg(a.m, s);
    const long long Mrr2 = Mrr - o_r - i_r - l, Mrs2 = Mrs + i_r - o_s, Msr2 = Msr + o_r - i_s;
    const long long dr2 = dr - kout - kin, ds2 = ds + kout + kin;
    const double Bd = (double)B;
    // phase B: the owner of each unique t adds its terms
    const double *__restrict__ fh = a.m.fh;
    const float *__restrict__ fl = a.m.fl;
    const double *__restrict__ rcp = a.m.rcp;
    double accS = 0.0, pf = 0.0, pb = 0.0;
    for (int j = gt; j < deg; j += G) {
        const bool out = j < nout;
        const int nb = out ? __ldg(a.col + ro + j) : __ldg(a.cscsrc + ci + j - nout);
        if (nb == v) continue;
        const int t = __ldg(a.b + nb);
        const int sl = tab_find(tab, log2cap, t);
        const int4 e = tab[sl];
        if (e.w != j) continue;
        const long long ot = e.y, it = e.z;
        const double c = (double)(ot + it);
        if (t == r) {
            pf += c * (double)(Mrs + Msr + 1) * __ldg(rcp + r);
            pb += c * (double)(2 * Mrr2 + 1) / ((double)dr2 + Bd);
        } else if (t == s) {
            pf += c * (double)(2 * Mss + 1) * __ldg(rcp + s);
            pb += c * (double)(Msr2 + Mrs2 + 1) / ((double)ds2 + Bd);
        } else {
            const long long Mrt = bm_at(a.m, r, t), Mst = bm_at(a.m, s, t);
            const long long Mtr = bm_at(a.m, t, r), Mts = bm_at(a.m, t, s);
            const double rt = __ldg(rcp + t);
            accS -= df_t(fh, fl, Mrt, -ot) + df_t(fh, fl, Mst, ot) + df_t(fh, fl, Mtr, -it) + df_t(fh, fl, Mts, it);
            pf += c * (double)(Mts + Mst + 1) * rt;
            pb += c * (double)(Mtr - it + Mrt - ot + 1) * rt;
        }
    }
    // the 2x2 core, the four degree terms and the self-loop terms, one per thread
    if (gt < 10) {
        switch (gt) {
            case 0: accS -= df_t(fh, fl, Mrr, -(o_r + i_r + l)); break;
            case 1: accS -= df_t(fh, fl, Mrs, i_r - o_s); break;
            case 2: accS -= df_t(fh, fl, Msr, o_r - i_s); break;
            case 3: accS -= df_t(fh, fl, Mss, o_s + i_s + l); break;
            case 4: accS += df_t(fh, fl, __ldg(a.m.dout + r), -kout); break;
            case 5: accS += df_t(fh, fl, __ldg(a.m.dout + s), kout); break;
            case 6: accS += df_t(fh, fl, __ldg(a.m.din + r), -kin); break;
            case 7: accS += df_t(fh, fl, __ldg(a.m.din + s), kin); break;
            case 8: if (l > 0) pf += 2.0 * (double)l * (double)(Mrs + Msr + 1) * __ldg(rcp + r); break;
            default: if (l > 0) pb += 2.0 * (double)l * (double)(Msr2 + Mrs2 + 1) / ((double)ds2 + Bd); break;
        }
    }
    const double dS = group_sum<G>(accS, sh);
    pf = group_sum<G>(pf, sh);
    pb = group_sum<G>(pb, sh);
    const double H = (kout + kin == 0) ? 1.0 : pb / pf;
    const double p = exp(-a.beta * dS) * H;
    const double u = ((double)w.w + 0.5) * (1.0 / 4294967296.0);
    dS_out = dS;
    H_out = H;
    acc_out = u <= p;
}

template <int G>
GSAP_DEV void tab_clear(int4 *tab, int slots, int gt) {
    for (int i = gt; i < slots; i += G) tab[i] = make_int4(-1, 0, 0, 0x7fffffff);
}

template <int G, bool WEIGHTED>
GSAP_DEV void do_vertex(const MoveArgs &a, int mode, int v, int4 *tab, int log2cap, int gt, double *sh,
                        int *bcast) {
    const int i = v - a.first;
    const uint32_t itr = a.itr_ptr ? __ldg(a.itr_ptr) : a.itr;
    const uint4 w = draws(a.seed, (uint32_t)v, 0u, itr, a.outer, 1u);
    int s;
    if (mode == MOVE_DELTA) {
        s = a.s_in[i];
    } else {
        if (G == 32) {
            s = propose_move<WEIGHTED>(a, v, w);
        } else {
            if ((threadIdx.x >> 5) == 0) {
                const int sp = propose_move<WEIGHTED>(a, v, w);
                if (threadIdx.x == 0) *bcast = sp;
            }
            __syncthreads();
            s = *bcast;
            __syncthreads();
        }
        if (a.s_out && gt == 0) a.s_out[i] = s;
        if (mode == MOVE_PROPOSE) return;
    }
    const int r = __ldg(a.b + v);
    double dS = 0.0, H = 1.0;
    bool acc = false;
    if (s != r) eval_move<G, WEIGHTED>(a, v, s, w, tab, log2cap, gt, sh, dS, H, acc);
    if (gt == 0) {
        if (a.dS) a.dS[i] = dS;
        if (a.H) a.H[i] = H;
        if (a.acc) a.acc[i] = acc ? 1 : 0;
    }
}

// One launch, two roles: CTAs [0, nbig_ctas) take the vertices of a.list
// (whose neighbour-block count can exceed 128) one CTA per vertex; the other
// CTAs take every other vertex of [first, first + count) one warp per vertex.
// The shared memory is the 8 warp tables, or one CTA table over the same bytes.
template <bool WEIGHTED>
__global__ void __launch_bounds__(MOVE_WARPS * 32, 3) k_move(MoveArgs a, int mode) {
    __shared__ int4 tabs[MOVE_WARPS * WARP_TAB];
    __shared__ double sh[MOVE_WARPS];
    __shared__ int bcast;
    const int wl = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if ((int)blockIdx.x < a.nbig_ctas) {
        int4 *tab = a.gtab ? a.gtab + ((size_t)blockIdx.x << a.gtab_log2) : tabs;
        const int log2cap = a.gtab_log2;
        for (int li = blockIdx.x; li < a.list_count; li += a.nbig_ctas) {
            const int v = a.list[li];
            tab_clear<CTA_THREADS>(tab, 1 << log2cap, threadIdx.x);
            __syncthreads();
            do_vertex<CTA_THREADS, WEIGHTED>(a, mode, v, tab, log2cap, threadIdx.x, sh, &bcast);
            __syncthreads();
        }
        return;
    }
    int4 *tab = tabs + wl * WARP_TAB;
    tab_clear<32>(tab, WARP_TAB, lane);
    __syncwarp();
    const int nwarps = (gridDim.x - a.nbig_ctas) * MOVE_WARPS;
    const bool skip_big = a.B > BIG_THR;
    for (int i = (blockIdx.x - a.nbig_ctas) * MOVE_WARPS + wl; i < a.count; i += nwarps) {
        const int v = a.first + i;
        // adjacency entries bound the number of unique neighbour blocks
        if (skip_big &&
            (__ldg(a.rowptr + v + 1) - __ldg(a.rowptr + v)) + (__ldg(a.cscptr + v + 1) - __ldg(a.cscptr + v)) > BIG_THR)
            continue;
        do_vertex<32, WEIGHTED>(a, mode, v, tab, WARP_TAB_LOG2, lane, nullptr, nullptr);
        __syncwarp();
        tab_clear<32>(tab, WARP_TAB, lane);
        __syncwarp();
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
    a.m = c.bm();
    a.first = first;
    a.count = count;
    a.list = nullptr;
    a.list_count = 0;
    a.s_in = mode == MOVE_DELTA ? s : nullptr;
    a.s_out = mode == MOVE_DELTA ? nullptr : s;
    a.dS = dS; a.H = H; a.acc = acc;
    a.gtab = nullptr;
    a.gtab_log2 = 0;
    const int m = (int)mode;
    a.nbig_ctas = 0;
    if (c.B > BIG_THR && !c.h_big.empty()) {
        // the big vertices inside [first, first + count)
        const auto lo = std::lower_bound(c.h_big.begin(), c.h_big.end(), first);
        const auto hi = std::lower_bound(c.h_big.begin(), c.h_big.end(), first + count);
        const int nbig = (int)(hi - lo);
        if (nbig > 0) {
            a.list = c.big + (lo - c.h_big.begin());
            a.list_count = nbig;
            int kmax = 0;
            for (auto it = lo; it != hi; ++it) {
                const int v = *it;
                kmax = std::max(kmax, (c.h_rowptr[v + 1] - c.h_rowptr[v]) + (c.h_cscptr[v + 1] - c.h_cscptr[v]));
            }
            const int log2cap = std::max(log2_ceil(2LL * std::min(kmax, c.B)), 5);
            a.gtab_log2 = log2cap;
            a.nbig_ctas = std::min(nbig, BIG_CTAS_MAX);
            if ((1 << log2cap) > CTA_SMEM_SLOTS) {
                if (((size_t)a.nbig_ctas << log2cap) > c.big_table_slots)
                    throw Error{GSAP_ENOMEM, "big-vertex table too small"};
                a.gtab = reinterpret_cast<int4 *>(c.big_tables);
            }
        }
    }
    const long long need = ((long long)count + MOVE_WARPS - 1) / MOVE_WARPS;
    const int grid = a.nbig_ctas + (int)std::max<long long>(1, std::min<long long>(need, 148LL * 8));
    if (c.weighted) k_move<true><<<grid, MOVE_WARPS * 32, 0, c.stream>>>(a, m);
    else k_move<false><<<grid, MOVE_WARPS * 32, 0, c.stream>>>(a, m);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
    // algorithmic bytes: adjacency ids (+ weights),
    // row / column pointers, b[v], the outputs (s, dS, acc)
    const long long adj = (long long)(c.h_rowptr[first + count] - c.h_rowptr[first]) +
                          (c.h_cscptr[first + count] - c.h_cscptr[first]);
    const double bytes = (c.weighted ? 8.0 : 4.0) * adj + (16.0 + 4.0 + 13.0) * count;
    kc_end(c, c.k_move, ev, bytes);
}

// ---------------------------------------------------------------- apply --
constexpr int APPLY_CHUNK = 1024;

__global__ void __launch_bounds__(256) k_apply(int first, int count, const int *__restrict__ s,
                                               const unsigned char *__restrict__ acc,
                                               const double *__restrict__ dS, int *__restrict__ b,
                                               double *__restrict__ partials, int *__restrict__ nacc) {
    __shared__ double sh[8];
    const int base = blockIdx.x * APPLY_CHUNK;
    double sum = 0.0;
    int na = 0;
    for (int k = threadIdx.x; k < APPLY_CHUNK; k += 256) {
        const int i = base + k;
        if (i < count && acc[i]) {
            b[first + i] = s[i];
            sum += dS ? dS[i] : 0.0;
            ++na;
        }
    }
    na = warp_sum(na);
    if (nacc && (threadIdx.x & 31) == 0 && na) atomicAdd(nacc, na);
    sum = warp_sum(sum);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = sum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < 8; ++w) t += sh[w];
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

void launch_apply(Ctx &c, int first, int count, const int *s, const unsigned char *acc, const double *dS,
                  double *dsum, int *nacc) {
    if (count <= 0) return;
    const int nb = (count + APPLY_CHUNK - 1) / APPLY_CHUNK;
    k_apply<<<nb, 256, 0, c.stream>>>(first, count, s, acc, dS, c.b, c.partials, nacc);
    k_sum_partials<<<1, 256, 0, c.stream>>>(c.partials, nb, dsum, 1);
    c.launches += 2;
    GSAP_CHECK_LAUNCH();
}

}  // namespace gsap
