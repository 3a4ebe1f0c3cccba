// merge.cu -- the block-merge phase (P:67 2.1, P:141 3, P:166-170 3.2,
// P:211-232 3.3):
//   (a3) every block r draws num_proposals merge targets (Alg. 1, excluding r;
//        readings Z6, Z8) and evaluates Delta S of merging r into s in exact
//        form (Eq. 4-6 with the terms Z11/Z12 add):
//          dS = -sum_{t != r,s} [g(M_st, M_rt) + g(M_ts, M_tr)]
//               - [f(M_ss + M_sr + M_rs + M_rr) - f(M_ss) - f(M_sr) - f(M_rs) - f(M_rr)]
//               + g(dout_s, dout_r) + g(din_s, din_r),   g(a,c) = f(a+c) - f(a) - f(c),
//        where only t in the intersection of the two rows (columns) contribute:
//        a warp walks the shorter row and looks the other up (dense copy or
//        binary search);  best_r = argmin_j (first j wins ties, R:Z16);
//   (a4) the perform-merge, in an exact parallel form of the
//        sequential GraphChallenge loop: rank by
//        (dS_best, r); reject the max-rank edge of every cycle of r -> best_r
//        (pointer doubling with running max); apply the accepted edges of the
//        shortest rank prefix with K of them; roots by pointer jumping;
//        relabel to the ranks of the roots present in b (R:Z18).
#include <algorithm>

#include <cstdlib>

#include "internal.h"
#include "prims.cuh"

namespace gsap {

typedef unsigned long long u64;

constexpr int MERGE_WARPS = 8;
constexpr int MAX_P = 32;

GSAP_DEV int propose_merge(const BM &m, int r, uint32_t j, uint64_t seed, uint32_t outer) {
    const uint32_t B = (uint32_t)m.B;
    const uint4 w = draws(seed, (uint32_t)r, j, 0u, outer, 0u);
    const uint32_t K = (uint32_t)bm_deg(m, r);
    if (m.mt) {   // N4, Alg. 1 lines 2-10 with the shared table; an s = r outcome is redrawn
        if (K > 0) {
            const int u = __ldg(m.mt + r);
            if (!coin_random(w.y, B, (uint32_t)bm_deg(m, u))) {
                const int s = __ldg(m.mt + u);
                if (s >= 0 && s != r) return s;
            }
        }
        int s = (int)pick(w.z, B - 1);
        if (s >= r) ++s;
        return s;
    }
    if (K > 0) {
        const int u = bm_walk(m, r, (long long)pick(w.x, K), -1);
        const uint32_t du = (uint32_t)bm_deg(m, u);
        if (!coin_random(w.y, B, du)) {
            const uint32_t T = du - (uint32_t)bm_at(m, u, r) - (uint32_t)bm_at(m, r, u);
            if (T > 0) return bm_walk(m, u, (long long)pick(w.z, T), r);
        }
    }
    int s = (int)pick(w.z, B - 1);
    if (s >= r) ++s;
    return s;
}

// sum over t != r, s of g(M_a t, M_b t) over the intersection of line a and
// line b (rows of the CSR, or columns of the CSC): walk the shorter line,
// look the other one up in its hash table (or the dense copy)
GSAP_DEV double inter_sum(const BM &m, bool cols, int a, int b, int r, int s) {
    const int *__restrict__ ptr = cols ? m.colptr : m.rowptr;
    const int *__restrict__ end = cols ? m.colend : m.rowend;
    const int *__restrict__ idx = cols ? m.row : m.col;
    const int *__restrict__ cnt = cols ? m.ccnt : m.cnt;
    const int alo = __ldg(ptr + a), ahi = __ldg(end + a);
    const int blo = __ldg(ptr + b), bhi = __ldg(end + b);
    const bool walk_a = (ahi - alo) <= (bhi - blo);
    const int lo = walk_a ? alo : blo, hi = walk_a ? ahi : bhi, other = walk_a ? b : a;
    Line L{};
    if (!m.dense) L = cols ? col_line(m, other) : row_line(m, other);
    double acc = 0.0;
    for (int i = lo + (int)(threadIdx.x & 31); i < hi; i += 32) {
        const int t = __ldg(idx + i);
        if (t == r || t == s) continue;
        const int m1 = __ldg(cnt + i);
        const int m2 = cols ? col_at(m, L, other, t) : row_at(m, L, other, t);
        acc += g2_t(m.ft, m1, m2);
    }
    return acc;
}

GSAP_DEV double merge_delta(const BM &m, int r, int s) {
    // rows r, s (t in both supports): g(M_st, M_rt); columns r, s: g(M_ts, M_tr)
    double acc = inter_sum(m, false, r, s, r, s) + inter_sum(m, true, r, s, r, s);
    acc = warp_sum(acc);
    const long long Mss = bm_at(m, s, s), Msr = bm_at(m, s, r), Mrs = bm_at(m, r, s), Mrr = bm_at(m, r, r);
    // f(a+b+c+d) - f(a) - f(b) - f(c) - f(d), telescoped into g's
    const double core = g2_t(m.ft, Mss, Msr) + g2_t(m.ft, Mss + Msr, Mrs) +
                        g2_t(m.ft, Mss + Msr + Mrs, Mrr);
    const double deg = g2_t(m.ft, __ldg(m.dout + s), __ldg(m.dout + r)) +
                       g2_t(m.ft, __ldg(m.din + s), __ldg(m.din + r));
    return -acc - core + deg;
}

struct MergeArgs {
    BM m;
    uint64_t seed;
    uint32_t outer;
    int P, first, count;
    bool propose;
    int *s;          // [count * P] in (propose = false) or out (nullable)
    double *dS;      // [count * P] out, nullable
    int *best;       // [count] out, nullable
    double *dSbest;  // [count] out, nullable
};

__global__ void __launch_bounds__(MERGE_WARPS * 32) k_merge(MergeArgs a) {
    const int lane = threadIdx.x & 31;
    const int nwarps = gridDim.x * MERGE_WARPS;
    for (int i = blockIdx.x * MERGE_WARPS + (threadIdx.x >> 5); i < a.count; i += nwarps) {
        const int r = a.first + i;
        int sj = -1;
        if (lane < a.P) {
            sj = a.propose ? propose_merge(a.m, r, (uint32_t)lane, a.seed, a.outer) : a.s[(size_t)i * a.P + lane];
            if (a.propose && a.s) a.s[(size_t)i * a.P + lane] = sj;
        }
        if (!a.dS && !a.best && !a.dSbest) continue;   // proposals only
        int bs = -1;
        double bd = 0.0;
        for (int j = 0; j < a.P; ++j) {
            const int s = __shfl_sync(FULL, sj, j);
            const double d = merge_delta(a.m, r, s);
            if (lane == 0) {
                if (a.dS) a.dS[(size_t)i * a.P + j] = d;
                if (j == 0 || d < bd) {
                    bd = d;
                    bs = s;
                }
            }
        }
        if (lane == 0) {
            if (a.best) a.best[i] = bs;
            if (a.dSbest) a.dSbest[i] = bd;
        }
    }
}

// one warp per (block, proposal j) pair: the P proposals of a block are
// evaluated in parallel warps instead of one after another by the block's
// warp (at small B the whole phase was P sequential merge_delta chains long);
// the same proposal and merge_delta per pair, so the same bits.  Writes s and
// dS per pair (into the caller's arrays or the context's scratch); k_merge_best
// then takes the first argmin per block.
__global__ void __launch_bounds__(MERGE_WARPS * 32) k_merge_pairs(MergeArgs a, int *__restrict__ sbuf,
                                                                  double *__restrict__ dbuf) {
    const int lane = threadIdx.x & 31;
    const long long total = (long long)a.count * a.P;
    const long long nwarps = (long long)gridDim.x * MERGE_WARPS;
    for (long long t = (long long)blockIdx.x * MERGE_WARPS + (threadIdx.x >> 5); t < total; t += nwarps) {
        const int i = (int)(t / a.P), j = (int)(t - (long long)i * a.P);
        const int r = a.first + i;
        int s = 0;
        if (lane == 0) s = a.propose ? propose_merge(a.m, r, (uint32_t)j, a.seed, a.outer) : sbuf[t];
        s = __shfl_sync(FULL, s, 0);
        if (!a.dS && !a.best && !a.dSbest) {   // proposals only
            if (lane == 0) sbuf[t] = s;
            continue;
        }
        const double d = merge_delta(a.m, r, s);
        if (lane == 0) {
            if (a.propose) sbuf[t] = s;
            dbuf[t] = d;
        }
    }
}

// best proposal per block: the first j with the smallest dS (strict <, R:Z16)
__global__ void k_merge_best(int count, int P, const int *__restrict__ sbuf, const double *__restrict__ dbuf,
                             int *__restrict__ best, double *__restrict__ dSbest) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < count; i += gridDim.x * blockDim.x) {
        int bs = sbuf[(size_t)i * P];
        double bd = dbuf[(size_t)i * P];
        for (int j = 1; j < P; ++j) {
            const double d = dbuf[(size_t)i * P + j];
            if (d < bd) {
                bd = d;
                bs = sbuf[(size_t)i * P + j];
            }
        }
        if (best) best[i] = bs;
        if (dSbest) dSbest[i] = bd;
    }
}

// N4: block x's table entry = a weighted neighbour block of x (the walk of
// R:O.4 with its own Philox draw), -1 for a block without edges
__global__ void k_fill_mt(BM m, uint64_t seed, uint32_t j, uint32_t itr, const unsigned *itr_ptr, uint32_t outer,
                          uint32_t phase, int *__restrict__ mt) {
    const uint32_t it = itr_ptr ? __ldg(itr_ptr) : itr;
    for (int x = blockIdx.x * blockDim.x + threadIdx.x; x < m.B; x += gridDim.x * blockDim.x) {
        const uint32_t d = (uint32_t)bm_deg(m, x);
        const uint4 w = draws(seed, (uint32_t)x, j, it, outer, phase);
        mt[x] = d ? bm_walk(m, x, (long long)pick(w.x, d), -1) : -1;
    }
}

void launch_fill_mt(Ctx &c, uint32_t j, uint32_t itr, uint32_t outer, uint32_t phase, const unsigned *d_itr) {
    if (c.prm.proposal_mode != 1) return;
    BM m = c.bm();
    m.mt = nullptr;
    const int g = (int)std::min<long long>(((long long)c.B + 255) / 256, 148LL * 8);
    k_fill_mt<<<std::max(g, 1), 256, 0, c.stream>>>(m, c.prm.seed, j, itr, d_itr, outer, phase, c.mt);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
}

void launch_merge_props(Ctx &c, uint32_t outer, int first, int count, bool propose, int *s, double *dS,
                        int *best, double *dSbest) {
    if (count <= 0) return;
    if (c.prm.num_proposals < 1 || c.prm.num_proposals > MAX_P)
        throw Error{GSAP_EINVAL, "num_proposals must be in [1, 32]"};
    if (c.B < 2) throw Error{GSAP_ESTATE, "merge proposals need B >= 2"};
    cudaEvent_t ev = nullptr;
    kc_begin(c, c.k_merge, &ev);
    MergeArgs a;
    a.m = c.bm();
    a.seed = c.prm.seed;
    a.outer = outer;
    a.P = c.prm.num_proposals;
    a.first = first;
    a.count = count;
    a.propose = propose;
    a.s = s;
    a.dS = dS;
    a.best = best;
    a.dSbest = dSbest;
    static const bool block_warps = getenv("GSAP_MERGE_WARP") != nullptr;   // A/B: one warp per block
    if (block_warps) {
        const long long need = ((long long)count + MERGE_WARPS - 1) / MERGE_WARPS;
        const int grid = (int)std::min<long long>(need, 148LL * 16);
        k_merge<<<grid, MERGE_WARPS * 32, 0, c.stream>>>(a);
        ++c.launches;
    } else {
        int *sbuf = s ? s : c.s;              // [count * P]: the context's proposal / dS scratch
        double *dbuf = dS ? dS : c.dS;
        const long long need = ((long long)count * a.P + MERGE_WARPS - 1) / MERGE_WARPS;
        const int grid = (int)std::min<long long>(need, 148LL * 16);
        k_merge_pairs<<<grid, MERGE_WARPS * 32, 0, c.stream>>>(a, sbuf, dbuf);
        ++c.launches;
        if (best || dSbest) {
            k_merge_best<<<(int)std::min<long long>((count + 255) / 256, 148LL * 8), 256, 0, c.stream>>>(
                count, a.P, sbuf, dbuf, best, dSbest);
            ++c.launches;
        }
    }
    GSAP_CHECK_LAUNCH();
    // algorithmic bytes: each proposal reads rows / columns r and s (id + cnt)
    // once; estimated from the mean row length (nnz unknown on the host)
    const double mean_row = (double)std::min<long long>(c.E, (long long)c.B * c.B) / std::max(1, c.B);
    kc_end(c, c.k_merge, ev, (double)count * (double)a.P * 4.0 * 8.0 * mean_row);
}

// ----------------------------------------------------------- selection --
__global__ void k_sel_keys(int B, const double *__restrict__ dS, u64 *__restrict__ keys, int *__restrict__ ids) {
    for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < B; r += gridDim.x * blockDim.x) {
        double d = dS[r];
        if (d == 0.0) d = 0.0;   // -0.0 == +0.0
        u64 bits = (u64)__double_as_longlong(d);
        bits = (bits >> 63) ? ~bits : (bits | 0x8000000000000000ULL);
        keys[r] = bits;
        ids[r] = r;
    }
}

__global__ void k_sel_rank(int B, const int *__restrict__ sorted_ids, int *__restrict__ rank) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < B; i += gridDim.x * blockDim.x) rank[sorted_ids[i]] = i;
}

__global__ void k_sel_init(int B, const int *__restrict__ best, const int *__restrict__ rank, int *__restrict__ nxt,
                           int *__restrict__ mx, int *__restrict__ oncyc) {
    for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < B; r += gridDim.x * blockDim.x) {
        nxt[r] = best[r];
        mx[r] = rank[r];
        oncyc[r] = 0;
    }
}

// one doubling step: mx'(r) = max(mx(r), mx(nxt(r))), nxt'(r) = nxt(nxt(r))
__global__ void k_sel_double(int B, const int *__restrict__ nxt, const int *__restrict__ mx, int *__restrict__ nxt2,
                             int *__restrict__ mx2) {
    for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < B; r += gridDim.x * blockDim.x) {
        const int n = nxt[r];
        nxt2[r] = nxt[n];
        mx2[r] = max(mx[r], mx[n]);
    }
}

__global__ void k_sel_mark(int B, const int *__restrict__ nxt, int *__restrict__ oncyc) {
    for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < B; r += gridDim.x * blockDim.x) oncyc[nxt[r]] = 1;
}

// acc_in_rank[i] = 1 iff the edge of the block at rank i is not a rejected cycle edge
__global__ void k_sel_accepted(int B, const int *__restrict__ sorted_ids, const int *__restrict__ rank,
                               const int *__restrict__ mx, const int *__restrict__ oncyc, int *__restrict__ acc_rank) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < B; i += gridDim.x * blockDim.x) {
        const int r = sorted_ids[i];
        const bool rejected = oncyc[r] && mx[r] == rank[r];
        acc_rank[i] = rejected ? 0 : 1;
    }
}

// applied edges: accepted and inside the shortest rank prefix with K of them;
// nxt(r) = best[r] if applied else r.  incl = inclusive scan of acc_rank.
__global__ void k_sel_applied(int B, int K, const int *__restrict__ sorted_ids, const int *__restrict__ acc_rank,
                              const int *__restrict__ incl, const int *__restrict__ best, int *__restrict__ nxt) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < B; i += gridDim.x * blockDim.x) {
        const int r = sorted_ids[i];
        const bool applied = acc_rank[i] && incl[i] <= K;
        nxt[r] = applied ? best[r] : r;
    }
}

__global__ void k_jump(int B, const int *__restrict__ nxt, int *__restrict__ nxt2) {
    for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < B; r += gridDim.x * blockDim.x) nxt2[r] = nxt[nxt[r]];
}

__global__ void k_present(int V, const int *__restrict__ b, const int *__restrict__ root, int *__restrict__ present) {
    for (int v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) present[root[b[v]]] = 1;
}

__global__ void k_labels(int B, const int *__restrict__ root, const int *__restrict__ present,
                         const int *__restrict__ excl, int *__restrict__ label) {
    for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < B; r += gridDim.x * blockDim.x) {
        const int x = root[r];
        label[r] = present[x] ? excl[x] : -1;
    }
}

__global__ void k_relabel(int V, const int *__restrict__ label, int *__restrict__ b) {
    for (int v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) b[v] = label[b[v]];
}

static inline int g256(long long n) { return (int)std::max<long long>(1, std::min<long long>((n + 255) / 256, 148LL * 32)); }

// ------------------------------------------- selection, one CTA (small B) --
// The block part of select_merges for B <= SEL_SMALL_B in ONE 1024-thread CTA
// (shared memory): the same keys (canonical dS bits, id), a bitonic sort on
// (key, id) -- the order of the stable radix sort --, the same pointer
// doubling with running max, cycle marks, accepted flags, inclusive scan,
// applied edges and pointer jumping; writes the roots.  Integer work only: the
// same result as the multi-kernel path, in one launch instead of ~2 log2(2B) + 20.
constexpr int SEL_SMALL_B = 4096;
constexpr int SEL_THREADS = 1024;

GSAP_DEV void sel_cta_scan_incl(int *a, int n, int *sh) {   // in place, inclusive, n <= SEL_SMALL_B
    const int per = (n + SEL_THREADS - 1) / SEL_THREADS;     // <= 4
    const int lo = threadIdx.x * per, hi = min(n, lo + per);
    int sum = 0;
    for (int i = lo; i < hi; ++i) sum += a[i];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int x = warp_incl_scan(sum);
    if (lane == 31) sh[w] = x;
    __syncthreads();
    if (w == 0) {
        const int y = warp_incl_scan(sh[lane]);
        sh[lane] = y;
    }
    __syncthreads();
    int run = (w ? sh[w - 1] : 0) + x - sum;
    for (int i = lo; i < hi; ++i) {
        run += a[i];
        a[i] = run;
    }
    __syncthreads();
}

__global__ void __launch_bounds__(SEL_THREADS) k_select_small(int B, int K, int rounds, const int *__restrict__ best,
                                                              const double *__restrict__ dS, int *__restrict__ root) {
    extern __shared__ __align__(16) unsigned char sel_raw[];
    u64 *key = reinterpret_cast<u64 *>(sel_raw);                 // [N]
    int *id = reinterpret_cast<int *>(key + SEL_SMALL_B);         // [N]
    int *rank = id + SEL_SMALL_B;                                 // [B]
    int *n0 = rank + SEL_SMALL_B, *n1 = n0 + SEL_SMALL_B;         // [B] x 2
    int *m0 = n1 + SEL_SMALL_B, *m1 = m0 + SEL_SMALL_B;           // [B] x 2
    int *flag = m1 + SEL_SMALL_B;                                 // [B]
    int *sh = flag + SEL_SMALL_B;                                 // [32]
    const int tid = threadIdx.x;
    int N = 1;
    while (N < B) N <<= 1;
    for (int r = tid; r < N; r += SEL_THREADS) {
        if (r < B) {
            double d = dS[r];
            if (d == 0.0) d = 0.0;   // -0.0 == +0.0
            u64 bits = (u64)__double_as_longlong(d);
            bits = (bits >> 63) ? ~bits : (bits | 0x8000000000000000ULL);
            key[r] = bits;
            id[r] = r;
        } else {
            key[r] = ~0ULL;
            id[r] = 0x7fffffff;
        }
    }
    __syncthreads();
    // bitonic sort of (key, id) ascending
    for (int k = 2; k <= N; k <<= 1) {
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = tid; i < (N >> 1); i += SEL_THREADS) {
                const int lo = ((i & ~(j - 1)) << 1) | (i & (j - 1)), hi = lo + j;
                const bool up = (lo & k) == 0;
                const u64 ka = key[lo], kb = key[hi];
                const int ia = id[lo], ib = id[hi];
                const bool gt = ka > kb || (ka == kb && ia > ib);
                if (gt == up) {
                    key[lo] = kb; key[hi] = ka;
                    id[lo] = ib; id[hi] = ia;
                }
            }
            __syncthreads();
        }
    }
    for (int i = tid; i < B; i += SEL_THREADS) rank[id[i]] = i;
    __syncthreads();
    for (int r = tid; r < B; r += SEL_THREADS) {
        n0[r] = best[r];
        m0[r] = rank[r];
        flag[r] = 0;   // oncyc
    }
    __syncthreads();
    for (int q = 0; q < rounds; ++q) {
        for (int r = tid; r < B; r += SEL_THREADS) {
            const int n = n0[r];
            n1[r] = n0[n];
            m1[r] = max(m0[r], m0[n]);
        }
        __syncthreads();
        int *t = n0; n0 = n1; n1 = t;
        t = m0; m0 = m1; m1 = t;
    }
    for (int r = tid; r < B; r += SEL_THREADS) flag[n0[r]] = 1;   // on a cycle
    __syncthreads();
    // accepted flags by rank (into n1: free now), then their inclusive scan
    for (int i = tid; i < B; i += SEL_THREADS) {
        const int r = id[i];
        n1[i] = (flag[r] && m0[r] == rank[r]) ? 0 : 1;
    }
    __syncthreads();
    for (int i = tid; i < B; i += SEL_THREADS) m1[i] = n1[i];
    __syncthreads();
    sel_cta_scan_incl(m1, B, sh);
    for (int i = tid; i < B; i += SEL_THREADS) {
        const int r = id[i];
        n0[r] = (n1[i] && m1[i] <= K) ? best[r] : r;
    }
    __syncthreads();
    for (int q = 0; q < rounds; ++q) {
        for (int r = tid; r < B; r += SEL_THREADS) flag[r] = n0[n0[r]];
        __syncthreads();
        for (int r = tid; r < B; r += SEL_THREADS) n0[r] = flag[r];
        __syncthreads();
    }
    for (int r = tid; r < B; r += SEL_THREADS) root[r] = n0[r];
}

// labels for B <= SEL_SMALL_B in one CTA: exclusive scan of `present`, new B,
// label[r] = rank of root(r) among the present roots (or -1)
__global__ void __launch_bounds__(SEL_THREADS) k_labels_small(int B, const int *__restrict__ root,
                                                              const int *__restrict__ present,
                                                              int *__restrict__ label, int *__restrict__ newB) {
    __shared__ int ex[SEL_SMALL_B + 1];
    __shared__ int sh[32];
    for (int r = threadIdx.x; r < B; r += SEL_THREADS) ex[r] = present[r];
    __syncthreads();
    sel_cta_scan_incl(ex, B, sh);
    for (int r = threadIdx.x; r < B; r += SEL_THREADS) {
        const int x = root[r];
        label[r] = present[x] ? ex[x] - 1 : -1;   // inclusive - 1 = exclusive (present[x] = 1)
    }
    if (threadIdx.x == 0) *newB = ex[B - 1];
}

static void select_merges_small(Ctx &c, const int *best, const double *dS, int K, int rounds) {
    const int B = c.B, V = c.V;
    const size_t smem = sizeof(u64) * SEL_SMALL_B + sizeof(int) * (7 * SEL_SMALL_B + 32);
    per_device((const void *)k_select_small, [&] {
        GSAP_CUDA(cudaFuncSetAttribute(k_select_small, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        return 1;
    });
    k_select_small<<<1, SEL_THREADS, smem, c.stream>>>(B, K, rounds, best, dS, c.nxt0);
    GSAP_CUDA(cudaMemsetAsync(c.present, 0, sizeof(int) * ((size_t)B + 1), c.stream));
    k_present<<<g256(V), 256, 0, c.stream>>>(V, c.b, c.nxt0, c.present);
    k_labels_small<<<1, SEL_THREADS, 0, c.stream>>>(B, c.nxt0, c.present, c.label, c.scal_i);
    k_relabel<<<g256(V), 256, 0, c.stream>>>(V, c.label, c.b);
    b_changed(c);
    c.launches += 4;
    GSAP_CHECK_LAUNCH();
}


void select_merges(Ctx &c, const int *best, const double *dS, int K, int *label_out) {
    Launcher L{c.stream, &c.launches};
    const int B = c.B, V = c.V;
    int rounds = 1;
    while ((1LL << rounds) < 2LL * B) ++rounds;
    if (B <= SEL_SMALL_B && c.prm.sel_small) {
        select_merges_small(c, best, dS, K, rounds);
        if (label_out)
            GSAP_CUDA(cudaMemcpyAsync(label_out, c.label, sizeof(int) * (size_t)B, cudaMemcpyDefault, c.stream));
        GSAP_CUDA(cudaMemcpyAsync(c.h_int, c.scal_i, sizeof(int), cudaMemcpyDeviceToHost, c.stream));
        GSAP_CUDA(cudaStreamSynchronize(c.stream));
        c.B = *c.h_int;
        return;
    }
    k_sel_keys<<<g256(B), 256, 0, c.stream>>>(B, dS, c.skey0, c.sval0);
    ++c.launches;
    const int w = radix_sort<u64, int, true>(c.skey0, c.skey1, c.sval0, c.sval1, nullptr, B, 64, c.counts,
                                             c.scan_tmp, L);
    const int *sorted = w ? c.sval1 : c.sval0;
    k_sel_rank<<<g256(B), 256, 0, c.stream>>>(B, sorted, c.sel_rank);
    k_sel_init<<<g256(B), 256, 0, c.stream>>>(B, best, c.sel_rank, c.nxt0, c.mx0, c.oncyc);
    c.launches += 2;
    int *n0 = c.nxt0, *n1 = c.nxt1, *m0 = c.mx0, *m1 = c.mx1;
    for (int k = 0; k < rounds; ++k) {
        k_sel_double<<<g256(B), 256, 0, c.stream>>>(B, n0, m0, n1, m1);
        std::swap(n0, n1);
        std::swap(m0, m1);
    }
    k_sel_mark<<<g256(B), 256, 0, c.stream>>>(B, n0, c.oncyc);
    k_sel_accepted<<<g256(B), 256, 0, c.stream>>>(B, sorted, c.sel_rank, m0, c.oncyc, c.flags);
    c.launches += rounds + 2;
    device_scan<int>(c.flags, c.pos, nullptr, B, true, c.scan_tmp, nullptr, L);
    k_sel_applied<<<g256(B), 256, 0, c.stream>>>(B, K, sorted, c.flags, c.pos, best, c.nxt0);
    ++c.launches;
    n0 = c.nxt0;
    n1 = c.nxt1;
    for (int k = 0; k < rounds; ++k) {
        k_jump<<<g256(B), 256, 0, c.stream>>>(B, n0, n1);
        std::swap(n0, n1);
    }
    c.launches += rounds;
    GSAP_CUDA(cudaMemsetAsync(c.present, 0, sizeof(int) * ((size_t)B + 1), c.stream));
    k_present<<<g256(V), 256, 0, c.stream>>>(V, c.b, n0, c.present);
    ++c.launches;
    device_scan<int>(c.present, c.pos, nullptr, B, false, c.scan_tmp, c.scal_i, L);
    k_labels<<<g256(B), 256, 0, c.stream>>>(B, n0, c.present, c.pos, c.label);
    k_relabel<<<g256(V), 256, 0, c.stream>>>(V, c.label, c.b);
    b_changed(c);
    c.launches += 2;
    GSAP_CHECK_LAUNCH();
    if (label_out)
        GSAP_CUDA(cudaMemcpyAsync(label_out, c.label, sizeof(int) * (size_t)B, cudaMemcpyDefault, c.stream));
    int newB = 0;
    GSAP_CUDA(cudaMemcpyAsync(c.h_int, c.scal_i, sizeof(int), cudaMemcpyDeviceToHost, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    newB = *c.h_int;
    c.B = newB;
}

}  // namespace gsap
