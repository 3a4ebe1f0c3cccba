// common.cuh -- device helpers shared by the GSAP sm_100a kernels.
//
// Philox4x32-10 (replaces the paper's cuRAND lookup tables, P:168 3.2 Fig. 4;
// reading Z6), the multiply-shift range map, the cancellation-free entropy
// differences used by Delta MDL (Eq. 3-7, P:205-246 3.3), warp reductions and
// blockmodel lookups.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#define GSAP_DEV __device__ __forceinline__

namespace gsap {

constexpr unsigned FULL = 0xffffffffu;

// ---------------------------------------------------------------- Philox --
// Random123 philox4x32 round: (hi(M1*c2)^c1^k0, lo(M1*c2), hi(M0*c0)^c3^k1, lo(M0*c0))
GSAP_DEV uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
    for (int i = 0; i < 10; ++i) {
        const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
        c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
        k.x += 0x9E3779B9u;
        k.y += 0xBB67AE85u;
    }
    return c;
}

// words for (id, draw, iteration, outer round, phase): ctr = (id, j, itr, outer<<1|phase)
GSAP_DEV uint4 draws(uint64_t seed, uint32_t id, uint32_t j, uint32_t itr, uint32_t outer,
                     uint32_t phase) {
    return philox4x32_10(make_uint4(id, j, itr, (outer << 1) | phase),
                         make_uint2((uint32_t)seed, (uint32_t)(seed >> 32)));
}

// floor(w * T / 2^32), T < 2^32
GSAP_DEV uint32_t pick(uint32_t w, uint32_t T) {
    return (uint32_t)(((uint64_t)w * (uint64_t)T) >> 32);
}

// the proposal coin x <= B / (B + d) as an exact integer test (reading Z9)
GSAP_DEV bool coin_random(uint32_t w1, uint32_t B, uint32_t d) {
    return (uint64_t)w1 * ((uint64_t)B + d) <= ((uint64_t)B << 32);
}

// ------------------------------------------------------------- entropy --
// f(m) = m ln m.  df(m, d) = f(m + d) - f(m) for integers m >= 0, m + d >= 0,
// without cancellation: d ln(m + d) + m log1p(d / m), the second term by its
// series when |d / m| <= 2^-7; below FT_N both f's come from a double-double
// table (written on the host in long double), so most terms need no
// transcendental at all.
constexpr int FT_N = 1 << 16;

GSAP_DEV double fx(double m) { return m > 0.0 ? m * log(m) : 0.0; }

GSAP_DEV double ftab(const double2 *__restrict__ ft, long long n) {
    const double2 e = __ldg(ft + n);
    return e.x + e.y;
}

GSAP_DEV double df_big(long long m, long long d) {
    const long long n = m + d;
    if (m == 0) return fx((double)n);
    if (n == 0) return -fx((double)m);
    const double x = (double)d / (double)m;
    double tail;
    if (fabs(x) <= 0.0078125) {
        // m log1p(x) = d (1 - x/2 + x^2/3 - x^3/4 + x^4/5 - x^5/6 + x^6/7 - x^7/8 + ...)
        double p = -1.0 / 8.0;
        p = fma(p, x, 1.0 / 7.0);
        p = fma(p, x, -1.0 / 6.0);
        p = fma(p, x, 1.0 / 5.0);
        p = fma(p, x, -1.0 / 4.0);
        p = fma(p, x, 1.0 / 3.0);
        p = fma(p, x, -1.0 / 2.0);
        tail = fma((double)d * x, p, (double)d);
    } else {
        tail = (double)m * log1p(x);
    }
    return fma((double)d, log((double)n), tail);
}

GSAP_DEV double df_t(const double2 *__restrict__ ft, long long m, long long d) {
    if (d == 0) return 0.0;
    const long long n = m + d;
    if (m < FT_N && n < FT_N) {
        const double2 a = __ldg(ft + n), b = __ldg(ft + m);
        return (a.x - b.x) + (a.y - b.y);
    }
    return df_big(m, d);
}

// g(a, c) = f(a + c) - f(a) - f(c) = a log1p(c/a) + c log1p(a/c)
GSAP_DEV double g2(long long a, long long c) {
    if (a == 0 || c == 0) return 0.0;
    return (double)a * log1p((double)c / (double)a) + (double)c * log1p((double)a / (double)c);
}

GSAP_DEV double g2_t(const double2 *__restrict__ ft, long long a, long long c) {
    if (a == 0 || c == 0) return 0.0;
    if (a + c < FT_N) {
        const double2 x = __ldg(ft + a + c), y = __ldg(ft + a), z = __ldg(ft + c);
        return ((x.x - y.x) - z.x) + ((x.y - y.y) - z.y);
    }
    return g2(a, c);
}

// -------------------------------------------------------------- warps --
GSAP_DEV unsigned lane_id() { return threadIdx.x & 31u; }

template <typename T>
GSAP_DEV T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}

GSAP_DEV int warp_incl_scan(int v) {
    const unsigned l = lane_id();
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(FULL, v, o);
        if (l >= (unsigned)o) v += t;
    }
    return v;
}

// ---------------------------------------------------------- blockmodel --
// CSR (rows ascending column) + CSC (columns ascending row), cum = inclusive
// prefix of cnt within a row / column, out/in degrees (P:143-162 3.1), and a
// dense row-major copy M[x*B+y] when B is small.
// Line x occupies [rowptr[x], rowend[x]): compact producers pass rowend =
// rowptr + 1; the multi-kernel sparse rebuild leaves each line in its
// counting-sort segment (padded CSR, cnt = 0 in the padding).
struct BM {
    int B;
    const int *__restrict__ dense;   // nullptr in the sparse regime
    const double2 *__restrict__ ft;  // f(m) = m ln m for m < FT_N, double-double {hi, lo}
    const double *__restrict__ rcp;  // 1 / (d_x + B) per block
    const int *__restrict__ rowptr;  // [B+1]
    const int *__restrict__ rowend;  // [B]: end of line x
    const int *__restrict__ col;
    const int *__restrict__ cnt;
    const int *__restrict__ cum;
    const int *__restrict__ colptr;  // [B+1]
    const int *__restrict__ colend;  // [B]
    const int *__restrict__ row;
    const int *__restrict__ ccnt;
    const int *__restrict__ ccum;
    const int *__restrict__ dout;
    const int *__restrict__ din;
    // N4 ablation (params.proposal_mode = 1, Alg. 1 P:180-200 with the
    // lookup tables of P:168 Fig. 4): one weighted neighbour block per block,
    // shared by every proposal of the phase / batch; nullptr otherwise
    const int *__restrict__ mt;
};

// the table's key: j word of the Philox counter of block x's table draw
// (MERGE: one table per merge phase; MOVE: one per batch, keyed by its first vertex)
constexpr uint32_t TABLE_J = 0x40000000u;

// first index i in [lo, hi) with a[i] > p (upper bound); hi if none
GSAP_DEV int upper_bound(const int *__restrict__ a, int lo, int hi, long long p) {
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if ((long long)__ldg(a + mid) > p) hi = mid;
        else lo = mid + 1;
    }
    return lo;
}

// one row (or column) of M, resolved once and searched many times: the
// lookups of a move all land in rows r, s and columns r, s, so the lines stay
// hot in L1 and a binary search costs a few cache hits
struct Line {
    const int *__restrict__ idx;
    const int *__restrict__ cnt;
    int len;
};

GSAP_DEV Line line_of(const int *__restrict__ idx, const int *__restrict__ cnt, const int *__restrict__ ptr,
                      const int *__restrict__ end, int x) {
    const int lo = __ldg(ptr + x);
    Line L;
    L.idx = idx + lo;
    L.cnt = cnt + lo;
    L.len = __ldg(end + x) - lo;
    return L;
}

GSAP_DEV int line_get(const Line &L, int y) {
    int a = 0, b = L.len;
    while (a < b) {
        const int mid = (a + b) >> 1;
        if (__ldg(L.idx + mid) < y) a = mid + 1;
        else b = mid;
    }
    return (a < L.len && __ldg(L.idx + a) == y) ? __ldg(L.cnt + a) : 0;
}

GSAP_DEV Line row_line(const BM &m, int x) { return line_of(m.col, m.cnt, m.rowptr, m.rowend, x); }
GSAP_DEV Line col_line(const BM &m, int y) { return line_of(m.row, m.ccnt, m.colptr, m.colend, y); }

GSAP_DEV int bm_at(const BM &m, int x, int y) {
    if (m.dense) return __ldg(m.dense + (size_t)x * m.B + y);
    return line_get(row_line(m, x), y);
}

// M_xy with row x resolved (sparse) / M_yx with column x resolved, dense fallback
GSAP_DEV int row_at(const BM &m, const Line &L, int x, int y) {
    return m.dense ? __ldg(m.dense + (size_t)x * m.B + y) : line_get(L, y);
}
GSAP_DEV int col_at(const BM &m, const Line &L, int x, int y) {   // M_{y x}
    return m.dense ? __ldg(m.dense + (size_t)y * m.B + x) : line_get(L, y);
}

// first index i in [lo, hi) with a[i] > p, whole warp (32-ary search: one
// dependent load per factor 32 of the range); hi if none.  Warp-uniform.
GSAP_DEV int warp_upper_bound(const int *__restrict__ a, int lo, int hi, long long p) {
    const int lane = (int)(threadIdx.x & 31);
    while (hi - lo > 32) {
        const int step = (hi - lo + 31) >> 5;
        const int idx = lo + lane * step;
        const bool gt = idx < hi && (long long)__ldg(a + idx) > p;
        const unsigned bal = __ballot_sync(FULL, gt);
        if (bal == 0) {
            const int last = min(31, (hi - 1 - lo) / step);
            lo = lo + last * step + 1;
        } else {
            const int f = __ffs(bal) - 1;   // a[lo + f*step] > p, a[lo + (f-1)*step] <= p
            const int nlo = f > 0 ? lo + (f - 1) * step + 1 : lo;
            hi = lo + f * step + 1;
            lo = nlo;
        }
    }
    const int idx = lo + lane;
    const unsigned bal = __ballot_sync(FULL, idx < hi && (long long)__ldg(a + idx) > p);
    return bal ? lo + __ffs(bal) - 1 : hi;
}

GSAP_DEV int bm_deg(const BM &m, int x) { return __ldg(m.dout + x) + __ldg(m.din + x); }

// the weighted neighbour block of u at offset p of (out-row u ++ in-col u),
// skipping id `skip` (-1: none) -- binary search on cum (R:O.4 step 4)
GSAP_DEV int bm_walk(const BM &m, int u, long long p, int skip) {
    const int rlo = __ldg(m.rowptr + u), rhi = __ldg(m.rowend + u);
    const int dout_u = __ldg(m.dout + u);
    int wskip = 0;
    if (skip >= 0) {
        int a = rlo, b = rhi;
        while (a < b) {
            const int mid = (a + b) >> 1;
            if (__ldg(m.col + mid) < skip) a = mid + 1;
            else b = mid;
        }
        if (a < rhi && __ldg(m.col + a) == skip) {
            wskip = __ldg(m.cnt + a);
            const long long before = (long long)__ldg(m.cum + a) - wskip;
            if (p >= before) p += wskip;
        }
    }
    if (p < dout_u) return __ldg(m.col + upper_bound(m.cum, rlo, rhi, p));
    long long q = p - dout_u;
    const int clo = __ldg(m.colptr + u), chi = __ldg(m.colend + u);
    if (skip >= 0) {
        int a = clo, b = chi;
        while (a < b) {
            const int mid = (a + b) >> 1;
            if (__ldg(m.row + mid) < skip) a = mid + 1;
            else b = mid;
        }
        if (a < chi && __ldg(m.row + a) == skip) {
            const int w = __ldg(m.ccnt + a);
            const long long before = (long long)__ldg(m.ccum + a) - w;
            if (q >= before) q += w;
        }
    }
    return __ldg(m.row + upper_bound(m.ccum, clo, chi, q));
}

// bm_walk without skipping, whole warp (MOVE proposals)
GSAP_DEV int bm_walk_warp(const BM &m, int u, long long p) {
    const int dout_u = __ldg(m.dout + u);
    if (p < dout_u) {
        const int i = warp_upper_bound(m.cum, __ldg(m.rowptr + u), __ldg(m.rowend + u), p);
        return __ldg(m.col + i);
    }
    const int i = warp_upper_bound(m.ccum, __ldg(m.colptr + u), __ldg(m.colend + u), p - dout_u);
    return __ldg(m.row + i);
}

}  // namespace gsap
