// rebuild.cu -- blockmodel rebuild (Alg. 2, P:248-283 3.4) and create-time
// graph preparation.
//
// M_xy = sum over edges u->w of weight [b_u = x][b_w = y] (P:56 2.1), stored
// as CSR (rows ascending column) + CSC (columns ascending row) with the
// in-row / in-column inclusive prefix `cum` used by the proposal walks, and the
// out / in block degrees.  Two regimes:
//   dense  (B^2 <= max(4E, 2^24)): shared-memory-privatised (B <= 221) or L2-atomic
//          histogram into a dense B x B matrix, tiled transpose, warp-per-row
//          compaction into CSR / CSC;
//   sparse (otherwise): counting sort of the edges by line + per-line segment
//          sort and run-length encoding (segsort.cuh), for rows (out-CSR) and
//          columns (in-CSC) alike.
#include <algorithm>
#include <cstdlib>

#include "internal.h"
#include "prims.cuh"
#include "segsort.cuh"
#include "coop.cuh"

namespace gsap {

typedef unsigned long long u64;

static inline int grid_for(long long n, int threads) {
    long long g = (n + threads - 1) / threads;
    return (int)(g < 1 ? 1 : (g > 2147483647LL ? 2147483647LL : g));
}

static inline int bits_for(long long n) {   // ceil(log2(n)), at least 1
    int b = 1;
    while ((1LL << b) < n) ++b;
    return b;
}

// ------------------------------------------------------------ create time --
__global__ void k_esrc_kout(int V, const int *__restrict__ rowptr, const int *__restrict__ col,
                            const int *__restrict__ wgt, int *__restrict__ esrc, int *__restrict__ kout,
                            int *__restrict__ selfw) {
    const int lane = threadIdx.x & 31;
    for (int v = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < V; v += (gridDim.x * blockDim.x) >> 5) {
        const int lo = rowptr[v], hi = rowptr[v + 1];
        int sum = 0, self = 0;
        for (int e = lo + lane; e < hi; e += 32) {
            esrc[e] = v;
            const int w = wgt ? wgt[e] : 1;
            sum += w;
            if (col[e] == v) self += w;
        }
        sum = warp_sum(sum);
        self = warp_sum(self);
        if (lane == 0) {
            kout[v] = sum;
            selfw[v] = self;
        }
    }
}

__global__ void k_csc_fill(int E, const int *__restrict__ idx, const int *__restrict__ esrc,
                           const int *__restrict__ wgt, int *__restrict__ cscsrc, int *__restrict__ cscwgt) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < E; i += (long long)gridDim.x * blockDim.x) {
        const int e = idx[i];
        cscsrc[i] = esrc[e];
        if (wgt) cscwgt[i] = wgt[e];
    }
}

__global__ void k_iota(int n, int *a) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        a[i] = (int)i;
}

// ptr[x] = first i in [0, n) with ids[i] >= x, x in [0, B]
template <typename T>
__global__ void k_ptr_from_ids(const T *__restrict__ ids, const int *d_n, int n_static, int B, int *__restrict__ ptr) {
    const int n = read_n(d_n, n_static);
    for (int x = blockIdx.x * blockDim.x + threadIdx.x; x <= B; x += gridDim.x * blockDim.x) {
        int lo = 0, hi = n;
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if ((long long)ids[mid] < (long long)x) lo = mid + 1;
            else hi = mid;
        }
        ptr[x] = lo;
    }
}

__global__ void k_invert(int n, const int *__restrict__ p, int *__restrict__ inv) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        inv[p[i]] = (int)i;
}

// the neighbour-block cache in full: nbo[p] = b[col[p]], nbi[q] = b[cscsrc[q]]
__global__ void k_nb_refresh(int E, const int *__restrict__ col, const int *__restrict__ cscsrc,
                             const int *__restrict__ b, int *__restrict__ nbo, int *__restrict__ nbi) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < E; i += (long long)gridDim.x * blockDim.x) {
        nbo[i] = __ldg(b + __ldg(col + i));
        nbi[i] = __ldg(b + __ldg(cscsrc + i));
    }
}

void nb_refresh(Ctx &c) {
    if (!c.nb_stale) return;
    c.nb_deferred = false;   // the full refresh covers the deferred update
    nb_join(c);
    if (c.E > 0) {
        const int g = (int)std::min<long long>(((long long)c.E + 255) / 256, 148LL * 16);
        k_nb_refresh<<<g, 256, 0, c.stream>>>(c.E, c.col, c.cscsrc, c.b, c.nbo, c.nbi);
        ++c.launches;
        GSAP_CHECK_LAUNCH();
    }
    c.nb_stale = false;
}

__global__ void k_kin(int V, const int *__restrict__ cscptr, const int *__restrict__ cscwgt, int *__restrict__ kin) {
    const int lane = threadIdx.x & 31;
    for (int v = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < V; v += (gridDim.x * blockDim.x) >> 5) {
        const int lo = cscptr[v], hi = cscptr[v + 1];
        int sum = 0;
        for (int e = lo + lane; e < hi; e += 32) sum += cscwgt ? cscwgt[e] : 1;
        sum = warp_sum(sum);
        if (lane == 0) kin[v] = sum;
    }
}

void build_graph_device(Ctx &c) {
    Launcher L{c.stream, &c.launches};
    const int V = c.V, E = c.E;
    k_esrc_kout<<<grid_for((long long)V * 32, 256), 256, 0, c.stream>>>(V, c.rowptr, c.col, c.wgt, c.esrc,
                                                                        c.kout, c.selfw);
    GSAP_CHECK_LAUNCH();
    ++c.launches;
    // CSC: stable sort of edge ids by destination (ties keep CSR order = by source)
    if (E > 0) {
        GSAP_CUDA(cudaMemcpyAsync(c.ukeys0, c.col, sizeof(int) * (size_t)E, cudaMemcpyDeviceToDevice, c.stream));
        k_iota<<<grid_for(E, 256), 256, 0, c.stream>>>(E, c.wa);
        ++c.launches;
        const int which = radix_sort<unsigned, int, true>(c.ukeys0, c.ukeys1, c.wa, c.wb, nullptr, E,
                                                          bits_for(V), c.counts, c.scan_tmp, L);
        const unsigned *keys = which ? c.ukeys1 : c.ukeys0;
        const int *idx = which ? c.wb : c.wa;
        k_csc_fill<<<grid_for(E, 256), 256, 0, c.stream>>>(E, idx, c.esrc, c.wgt, c.cscsrc, c.cscwgt);
        k_ptr_from_ids<unsigned><<<grid_for(V + 1, 256), 256, 0, c.stream>>>(keys, nullptr, E, V, c.cscptr);
        // position maps of the neighbour-block cache: CSC position q holds CSR edge idx[q]
        GSAP_CUDA(cudaMemcpyAsync(c.csc2csr, idx, sizeof(int) * (size_t)E, cudaMemcpyDeviceToDevice, c.stream));
        k_invert<<<grid_for(E, 256), 256, 0, c.stream>>>(E, idx, c.csr2csc);
        c.launches += 3;
    } else {
        GSAP_CUDA(cudaMemsetAsync(c.cscptr, 0, sizeof(int) * ((size_t)V + 1), c.stream));
    }
    k_kin<<<grid_for((long long)V * 32, 256), 256, 0, c.stream>>>(V, c.cscptr, c.cscwgt, c.kin);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
}

// ----------------------------------------------------------------- dense --
bool dense_ok(const Ctx &c, int B) { return (size_t)B * (size_t)B <= c.dense_cap; }

constexpr int HIST_SMEM_MAX_B = 221;   // B^2 * 4 bytes <= 195 KB of shared memory

// histogram of (b[src], b[dst]) over an edge range; PRIV: privatised in smem
template <bool PRIV>
__global__ void __launch_bounds__(1024) k_hist(int E, const int *__restrict__ esrc, const int *__restrict__ nbo,
                                                const int *__restrict__ wgt, const int *__restrict__ b, int B,
                                                int *__restrict__ M) {
    extern __shared__ int h[];
    const int BB = B * B;
    if (PRIV) {
        for (int i = threadIdx.x; i < BB; i += blockDim.x) h[i] = 0;
        __syncthreads();
    }
    int *dst = PRIV ? h : M;
    const long long chunk = ((long long)E + gridDim.x - 1) / gridDim.x;
    const long long lo = (long long)blockIdx.x * chunk;
    const long long hi = min((long long)E, lo + chunk);
    // iterate whole warps so that __match_any_sync sees a converged warp
    for (long long e0 = lo; e0 < hi; e0 += blockDim.x) {
        const long long e = e0 + threadIdx.x;
        int key = -1, w = 0;
        if (e < hi) {
            key = __ldg(b + __ldg(esrc + e)) * B + __ldg(nbo + e);
            w = wgt ? __ldg(wgt + e) : 1;
        }
        if (wgt) {
            if (key >= 0) atomicAdd(dst + key, w);
        } else {
            const unsigned peers = __match_any_sync(FULL, key);
            if (key >= 0 && (int)(threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(dst + key, __popc(peers));
        }
    }
    if (PRIV) {
        __syncthreads();
        for (int i = threadIdx.x; i < BB; i += blockDim.x) {
            const int v = h[i];
            if (v) atomicAdd(M + i, v);
        }
    }
}

__global__ void k_transpose(const int *__restrict__ M, int B, int *__restrict__ T) {
    __shared__ int tile[32][33];
    const int bx = blockIdx.x * 32, by = blockIdx.y * 32;
    for (int j = threadIdx.y; j < 32; j += blockDim.y) {
        const int x = by + j, y = bx + threadIdx.x;
        tile[j][threadIdx.x] = (x < B && y < B) ? M[(size_t)x * B + y] : 0;
    }
    __syncthreads();
    for (int j = threadIdx.y; j < 32; j += blockDim.y) {
        const int x = bx + j, y = by + threadIdx.x;
        if (x < B && y < B) T[(size_t)x * B + y] = tile[threadIdx.x][j];
    }
}



// ------------------------------------------------ dense, one kernel --
// The whole dense rebuild as ONE persistent cooperative kernel (params.dense_coop).
// The multi-kernel path (memset, histogram, transpose, stats, scan,
// compaction) is six launches of a few microseconds of work each at the B of
// the late rounds; here they are phases separated by grid barriers:
//   SMEM (B <= 221: the B x B histogram fits one CTA's shared memory)
//     P1 every CTA histograms a contiguous edge chunk (four edges per thread
//        per step, 16-byte loads, match_any aggregation) in shared memory and
//        adds its non-zeros into `acc` (zero on entry); line stats zeroed | barrier
//     P2 one warp per row x: M[x][.] = acc[x][.] (acc row re-zeroed for the
//        next call), Mt[.][x], row non-zeros and dout; column non-zeros and
//        din by integer atomics                                           | barrier
//     P3 one warp per line (rows of M, then rows of Mt = columns of M): its
//        offset = sum of the preceding lines' non-zeros, then the compaction
//        (idx, cnt, in-line prefix cum) and rcp = 1 / (d + B).
//   global (221 < B, B^2 <= dense_cap)
//     P0 zero M and the line stats                                        | barrier
//     P1 the same edge loop with L2 atomics straight into M                | barrier
//     P2 one warp per 32 x 32 tile of M: 32 independent loads, Mt through a
//        shared-memory tile, line non-zeros and sums by atomics            | barrier
//     P2b CTA 0 / 1 scan the row / column non-zeros into the pointers      | barrier
//     P3 compaction at the scanned offsets.
// Integer arithmetic throughout: the same bits as rebuild_dense.
constexpr int DC_THREADS = 512;
constexpr int DC_WARPS = DC_THREADS / 32;
constexpr size_t DC_TILE_SMEM = sizeof(int) * DC_WARPS * 32 * 33;

struct DenseArgs {
    int E, B;
    const int *__restrict__ esrc;
    const int *__restrict__ col;
    const int *__restrict__ wgt;
    const int *__restrict__ b;
    int *acc, *M, *Mt, *rownnz, *colnnz, *dout, *din;
    int *ptrA, *idxA, *cntA, *cumA, *ptrB, *idxB, *cntB, *cumB;
    double *rcp;
    int *d_nnz;
    unsigned *bar;
    const int *skip;   // N2: the batch's moved-vertex count (nullable); 0 = the blockmodel is unchanged
};

// exclusive scan of in[0, n) into out[0, n], out[n] = total, by one CTA of DC_THREADS
GSAP_DEV void dc_cta_scan(const int *in, int *out, int n, int *sh) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int carry = 0;
    for (int base = 0; base < n; base += DC_THREADS * 8) {
        int v[8], sm = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int idx = base + threadIdx.x * 8 + i;
            v[i] = idx < n ? __ldcg(in + idx) : 0;
            sm += v[i];
        }
        const int x = warp_incl_scan(sm);
        if (lane == 31) sh[w] = x;
        __syncthreads();
        int wb = 0, tot = 0;
        for (int i = 0; i < DC_WARPS; ++i) {
            const int q = sh[i];
            if (i < w) wb += q;
            tot += q;
        }
        __syncthreads();
        int ex = carry + wb + x - sm;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int idx = base + threadIdx.x * 8 + i;
            if (idx < n) out[idx] = ex;
            ex += v[i];
        }
        carry += tot;
    }
    if (threadIdx.x == 0) out[n] = carry;
}

template <bool SMEM>
__global__ void __launch_bounds__(DC_THREADS) k_rebuild_dense(DenseArgs a) {
    if (a.skip && *a.skip == 0) return;   // every CTA returns before any grid barrier
    extern __shared__ int h[];
    const int B = a.B, E = a.E;
    const size_t BB = (size_t)B * B;
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x, gthreads = gridDim.x * blockDim.x;
    const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5, gwarp = gtid >> 5, gwarps = gthreads >> 5;
    int *hist = SMEM ? h : a.M;
    // P0 / P1: line stats zeroed (read again after the next barrier)
    for (int i = gtid; i < B; i += gthreads) {
        a.rownnz[i] = 0;
        a.colnnz[i] = 0;
        a.dout[i] = 0;
        a.din[i] = 0;
    }
    if (SMEM) {
        for (int i = threadIdx.x; i < (int)BB; i += blockDim.x) h[i] = 0;
        __syncthreads();
    } else {
        int4 *M4 = reinterpret_cast<int4 *>(a.M);
        const size_t n4 = BB >> 2;
        for (size_t i = gtid; i < n4; i += gthreads) M4[i] = make_int4(0, 0, 0, 0);
        for (size_t i = (n4 << 2) + gtid; i < BB; i += gthreads) a.M[i] = 0;
        grid_sync(a.bar);
    }
    // P1: histogram of (b[src], b[dst]) over a contiguous edge chunk per CTA
    const long long chunk = ((((long long)E + gridDim.x - 1) / gridDim.x) + 3) & ~3LL;
    const long long lo = (long long)blockIdx.x * chunk;
    const long long hi = min((long long)E, lo + chunk);
    for (long long base = lo; base < hi; base += 4LL * blockDim.x) {   // uniform trip count per CTA
        const long long e0 = base + 4LL * threadIdx.x;
        int src[4], dst[4], w[4] = {1, 1, 1, 1};
        if (e0 + 3 < hi) {
            const int4 s4 = __ldg(reinterpret_cast<const int4 *>(a.esrc + e0));
            const int4 d4 = __ldg(reinterpret_cast<const int4 *>(a.col + e0));
            src[0] = s4.x; src[1] = s4.y; src[2] = s4.z; src[3] = s4.w;
            dst[0] = d4.x; dst[1] = d4.y; dst[2] = d4.z; dst[3] = d4.w;
            if (a.wgt) {
                const int4 w4 = __ldg(reinterpret_cast<const int4 *>(a.wgt + e0));
                w[0] = w4.x; w[1] = w4.y; w[2] = w4.z; w[3] = w4.w;
            }
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const bool ok = e0 + k < hi;
                src[k] = ok ? __ldg(a.esrc + e0 + k) : -1;
                dst[k] = ok ? __ldg(a.col + e0 + k) : -1;
                if (a.wgt) w[k] = ok ? __ldg(a.wgt + e0 + k) : 0;
            }
        }
        int key[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) key[k] = src[k] >= 0 ? __ldg(a.b + src[k]) * B + __ldg(a.b + dst[k]) : -1;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            if (a.wgt) {
                if (key[k] >= 0) atomicAdd(hist + key[k], w[k]);
            } else {
                const unsigned peers = __match_any_sync(FULL, key[k]);
                if (key[k] >= 0 && lane == __ffs(peers) - 1) atomicAdd(hist + key[k], __popc(peers));
            }
        }
    }
    if (SMEM) {
        __syncthreads();
        for (int i = threadIdx.x; i < (int)BB; i += blockDim.x) {
            const int v = h[i];
            if (v) atomicAdd(a.acc + i, v);
        }
    }
    grid_sync(a.bar);
    // P2 (SMEM, small B): one warp per row x -- M[x][.] = acc[x][.] (acc row
    // re-zeroed), Mt[.][x], row non-zeros / dout; columns by atomics
    if (SMEM) {
        for (int x = gwarp; x < B; x += gwarps) {
            int c = 0, sm = 0;
            for (int y = lane; y < B; y += 32) {
                const int v = __ldcg(a.acc + (size_t)x * B + y);
                a.acc[(size_t)x * B + y] = 0;
                a.M[(size_t)x * B + y] = v;
                a.Mt[(size_t)y * B + x] = v;
                if (v) {
                    ++c;
                    sm += v;
                    atomicAdd(a.colnnz + y, 1);
                    atomicAdd(a.din + y, v);
                }
            }
            c = __reduce_add_sync(FULL, c);
            sm = __reduce_add_sync(FULL, sm);
            if (lane == 0) {
                a.rownnz[x] = c;
                a.dout[x] = sm;
            }
        }
    }
    // P2 (global, larger B): 32 x 32 tiles, one warp each
    if (!SMEM) {
        const int nt = (B + 31) >> 5;
        int *tile = h + wl * (32 * 33);   // the histogram's shared memory is free again
        const int *src = SMEM ? a.acc : a.M;
        for (int t = gwarp; t < nt * nt; t += gwarps) {
            const int x0 = (t / nt) << 5, y0 = (t % nt) << 5, y = y0 + lane;
            const int rows = min(32, B - x0);
            int v[32];
#pragma unroll
            for (int i = 0; i < 32; ++i)   // 32 independent loads in flight
                v[i] = (i < rows && y < B) ? __ldcg(src + (size_t)(x0 + i) * B + y) : 0;
            int cn = 0, cs = 0;
#pragma unroll
            for (int i = 0; i < 32; ++i) {
                if (SMEM && i < rows && y < B) {
                    const size_t at = (size_t)(x0 + i) * B + y;
                    a.M[at] = v[i];
                    a.acc[at] = 0;
                }
                tile[i * 33 + lane] = v[i];
                const int rn = __reduce_add_sync(FULL, v[i] != 0 ? 1 : 0);
                const int rs = __reduce_add_sync(FULL, v[i]);
                if (lane == i && rn) {   // row i's sums, one lane each
                    atomicAdd(a.rownnz + x0 + i, rn);
                    atomicAdd(a.dout + x0 + i, rs);
                }
                cn += v[i] != 0;
                cs += v[i];
            }
            if (y < B && cn) {
                atomicAdd(a.colnnz + y, cn);
                atomicAdd(a.din + y, cs);
            }
            __syncwarp();
            const int xx = x0 + lane;
            for (int i = 0; i < 32 && y0 + i < B; ++i)
                if (xx < B) a.Mt[(size_t)(y0 + i) * B + xx] = tile[lane * 33 + i];
            __syncwarp();
        }
    }
    grid_sync(a.bar);
    if (!SMEM) {   // P2b
        if (blockIdx.x < 2) {
            dc_cta_scan(blockIdx.x ? a.colnnz : a.rownnz, blockIdx.x ? a.ptrB : a.ptrA, B, h);
            if (blockIdx.x == 0 && threadIdx.x == 0) *a.d_nnz = a.ptrA[B];
        }
        grid_sync(a.bar);
    }
    // P3
    for (int x2 = gwarp; x2 < 2 * B; x2 += gwarps) {
        const bool t = x2 >= B;
        const int x = t ? x2 - B : x2;
        int *__restrict__ ptr = t ? a.ptrB : a.ptrA;
        int off;
        if (SMEM) {
            const int *nz = t ? a.colnnz : a.rownnz;
            off = 0;
            for (int y = lane; y < x; y += 32) off += __ldcg(nz + y);
            off = __reduce_add_sync(FULL, off);
            if (lane == 0) {
                ptr[x] = off;
                if (x == B - 1) {
                    const int tot = off + __ldcg(nz + x);
                    ptr[B] = tot;
                    if (!t) *a.d_nnz = tot;
                }
            }
        } else {
            off = __ldcg(ptr + x);
        }
        if (!t && lane == 0)
            a.rcp[x] = 1.0 / ((double)__ldcg(a.dout + x) + (double)__ldcg(a.din + x) + (double)B);
        const int *R = (t ? a.Mt : a.M) + (size_t)x * B;
        int *__restrict__ idx = t ? a.idxB : a.idxA;
        int *__restrict__ cnt = t ? a.cntB : a.cntA;
        int *__restrict__ cum = t ? a.cumB : a.cumA;
        int base = off, run = 0;
        int nxt[4];   // the next step's entries, loaded one step ahead
#pragma unroll
        for (int k = 0; k < 4; ++k) nxt[k] = 4 * lane + k < B ? __ldcg(R + 4 * lane + k) : 0;
        for (int y0 = 0; y0 < B; y0 += 128) {
            const int y = y0 + 4 * lane;
            int v[4], nzc = 0, s4 = 0;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                v[k] = nxt[k];
                nxt[k] = y + 128 + k < B ? __ldcg(R + y + 128 + k) : 0;
                nzc += v[k] != 0;
                s4 += v[k];
            }
            const int nzi = warp_incl_scan(nzc), smi = warp_incl_scan(s4);
            int p = base + nzi - nzc, sc = run + smi - s4;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                sc += v[k];
                if (v[k] != 0) {
                    idx[p] = y + k;
                    cnt[p] = v[k];
                    cum[p] = sc;
                    ++p;
                }
            }
            base += __shfl_sync(FULL, nzi, 31);
            run += __shfl_sync(FULL, smi, 31);
        }
    }
}

template <bool SMEM>
static void launch_rebuild_dense_coop(Ctx &c, const int *skip = nullptr) {
    DenseArgs a;
    a.skip = skip;
    a.E = c.E;
    a.B = c.B;
    a.esrc = c.esrc; a.col = c.col; a.wgt = c.wgt; a.b = c.b;   // b gathered: runs beside a pending cache update
    a.acc = c.small_acc; a.M = c.dense; a.Mt = c.denseT;
    a.rownnz = c.dnnz_r; a.colnnz = c.dnnz_c; a.dout = c.dout; a.din = c.din;   // kept for N2
    a.ptrA = c.bm_rowptr; a.idxA = c.bm_col; a.cntA = c.bm_cnt; a.cumA = c.bm_cum;
    a.ptrB = c.bm_colptr; a.idxB = c.bm_row; a.cntB = c.bm_ccnt; a.cumB = c.bm_ccum;
    a.rcp = c.rcp;
    a.d_nnz = c.d_nnz;
    a.bar = c.coop_bar;
    const size_t smem_max = SMEM ? std::max(DC_TILE_SMEM, sizeof(int) * SMALL_MAX_B * SMALL_MAX_B) : DC_TILE_SMEM;
    const int grid = per_device((const void *)k_rebuild_dense<SMEM>, [&] {
        GSAP_CUDA(cudaFuncSetAttribute(k_rebuild_dense<SMEM>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem_max));
        int per_sm = 0, sms = 0, dev = 0;
        GSAP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_rebuild_dense<SMEM>, DC_THREADS,
                                                                smem_max));
        GSAP_CUDA(cudaGetDevice(&dev));
        GSAP_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        return std::max(1, std::min(per_sm, SMEM ? 1 : 2) * sms);
    });
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(DC_THREADS);
    cfg.dynamicSmemBytes = SMEM ? std::max(DC_TILE_SMEM, sizeof(int) * (size_t)c.B * c.B) : DC_TILE_SMEM;
    cfg.stream = c.stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    GSAP_CUDA(cudaLaunchKernelEx(&cfg, k_rebuild_dense<SMEM>, a));
    ++c.launches;
}

// N2 (incremental blockmodel update, P:250-255 3.4, Fig. 6): the change of M
// (and of its transpose) by the batch's applied moves, instead of a histogram
// of every edge.  One warp per moved vertex v (old block r = oldb[v], new
// block s = b[v]); an edge u -> w changes from (old b_u, old b_w) to (new b_u,
// new b_w), each edge counted once: v's out-edges always, its in-edges only
// from vertices that did not move (a moved source covers the edge with its
// own out-edges; a self-loop is an out-edge).  Integer additions: the result
// equals the full histogram exactly.
__global__ void __launch_bounds__(256) k_dense_delta(const int *__restrict__ moved, const int *__restrict__ moved_cnt,
                                                     int first, int count, const unsigned char *__restrict__ acc,
                                                     const int *__restrict__ oldb, const int *__restrict__ b,
                                                     const int *__restrict__ rowptr, const int *__restrict__ col,
                                                     const int *__restrict__ wgt, const int *__restrict__ cscptr,
                                                     const int *__restrict__ cscsrc, const int *__restrict__ cscwgt,
                                                     int B, int *__restrict__ M, int *__restrict__ Mt,
                                                     unsigned char *__restrict__ dirty) {
    const int n = *moved_cnt;
    const int lane = threadIdx.x & 31;
    for (int k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < n; k += (gridDim.x * blockDim.x) >> 5) {
        const int v = moved[k];
        const int r = oldb[v], s = b[v];
        const int ro = rowptr[v], nout = rowptr[v + 1] - ro;
        const int ci = cscptr[v], nin = cscptr[v + 1] - ci;
        // padded layout (dirty != nullptr): every line whose entries change --
        // rows r, s (out-edges), columns r, s (in-edges), and the neighbours'
        // lines marked below
        if (dirty && lane == 0) {
            if (nout) dirty[r] = dirty[s] = 1;
            if (nin) dirty[B + r] = dirty[B + s] = 1;
        }
        for (int j = lane; j < nout; j += 32) {
            const int w = col[ro + j];
            const int wt = wgt ? wgt[ro + j] : 1;
            const int bn = b[w];
            const bool wm = w >= first && w < first + count && acc[w - first];
            const int bo = wm ? oldb[w] : bn;
            atomicAdd(M + (size_t)r * B + bo, -wt);
            atomicAdd(M + (size_t)s * B + bn, wt);
            atomicAdd(Mt + (size_t)bo * B + r, -wt);
            atomicAdd(Mt + (size_t)bn * B + s, wt);
            if (dirty) dirty[B + bo] = dirty[B + bn] = 1;
        }
        for (int j = lane; j < nin; j += 32) {
            const int w = cscsrc[ci + j];
            if (w >= first && w < first + count && acc[w - first]) continue;   // moved source (incl. v's self-loop)
            const int wt = cscwgt ? cscwgt[ci + j] : 1;
            const int bw = b[w];
            atomicAdd(M + (size_t)bw * B + r, -wt);
            atomicAdd(M + (size_t)bw * B + s, wt);
            atomicAdd(Mt + (size_t)r * B + bw, -wt);
            atomicAdd(Mt + (size_t)s * B + bw, wt);
            if (dirty) dirty[bw] = 1;
        }
    }
}

// the dense regime's lines in the PADDED layout (line x of M at x B, of Mt at
// x B in the column arrays; end[x] marks its last run, cnt is zero beyond it):
// one warp per line compacts the dense row (idx, cnt, in-line prefix cum) and
// writes its sum (dout / din); DIRTY: only the lines k_dense_delta marked
// (flag cleared), zeroing the counts its previous version left beyond the new
// end; else every line (counts pre-zeroed).  The last CTA to finish writes
// rcp = 1 / (d + B) for every block, the extent B^2 and the end pointer.
// Integer work: the same runs as the compact layout, at other offsets.
template <bool DIRTY>
__global__ void __launch_bounds__(256) k_dense_lines(const int *__restrict__ M, const int *__restrict__ Mt, int B,
                                                     unsigned char *__restrict__ dirty, int *__restrict__ ptrA,
                                                     int *__restrict__ endA, int *__restrict__ idxA,
                                                     int *__restrict__ cntA, int *__restrict__ cumA,
                                                     int *__restrict__ ptrB, int *__restrict__ endB,
                                                     int *__restrict__ idxB, int *__restrict__ cntB,
                                                     int *__restrict__ cumB, int *__restrict__ dout,
                                                     int *__restrict__ din, double *__restrict__ rcp,
                                                     int *__restrict__ d_nnz, unsigned *__restrict__ arrive,
                                                     const int *__restrict__ skip) {
    if (skip && *skip == 0) return;   // the batch moved nothing: every line as it was
    __shared__ bool last;
    // each warp stages its line DL_CH entries at a time: all the chunk's loads
    // in flight at once (one memory latency per 1024 entries instead of one
    // per 128-entry step), then the compaction from shared memory
    constexpr int DL_CH = 1024;
    __shared__ int4 stage[8][DL_CH / 4];
    const int lane = threadIdx.x & 31;
    int *sb = reinterpret_cast<int *>(stage[threadIdx.x >> 5]);
    for (int x2 = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; x2 < 2 * B; x2 += (gridDim.x * blockDim.x) >> 5) {
        if (DIRTY && !dirty[x2]) continue;   // warp-uniform
        const bool t = x2 >= B;
        const int x = t ? x2 - B : x2;
        const int *__restrict__ R = (t ? Mt : M) + (size_t)x * B;
        int *__restrict__ idx = t ? idxB : idxA;
        int *__restrict__ cnt = t ? cntB : cntA;
        int *__restrict__ cum = t ? cumB : cumA;
        int *__restrict__ end = t ? endB : endA;
        const int lo = x * B;
        const int old_end = DIRTY ? end[x] : lo;
        int base = lo, run = 0;
        for (int c0 = 0; c0 < B; c0 += DL_CH) {
            int tmp[DL_CH / 32];
#pragma unroll
            for (int j = 0; j < DL_CH / 32; ++j) {
                const int y = c0 + j * 32 + lane;
                tmp[j] = y < B ? __ldg(R + y) : 0;
            }
#pragma unroll
            for (int j = 0; j < DL_CH / 32; ++j) sb[j * 32 + lane] = tmp[j];
            __syncwarp();
            const int n = min(DL_CH, B - c0);
            for (int s0 = 0; s0 < n; s0 += 128) {
                const int y = c0 + s0 + 4 * lane;
                const int4 q4 = reinterpret_cast<const int4 *>(sb)[(s0 >> 2) + lane];
                const int v[4] = {q4.x, q4.y, q4.z, q4.w};   // zero beyond B
                int nz = 0, sm = 0;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    nz += v[k] != 0;
                    sm += v[k];
                }
                const int nzi = warp_incl_scan(nz), smi = warp_incl_scan(sm);
                int p = base + nzi - nz, sc = run + smi - sm;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    sc += v[k];
                    if (v[k] != 0) {
                        idx[p] = y + k;
                        cnt[p] = v[k];
                        cum[p] = sc;
                        ++p;
                    }
                }
                base += __shfl_sync(FULL, nzi, 31);
                run += __shfl_sync(FULL, smi, 31);
            }
            __syncwarp();   // the stage is rewritten by the next chunk
        }
        if (DIRTY)
            for (int q = base + lane; q < old_end; q += 32) cnt[q] = 0;   // the previous version's tail
        if (lane == 0) {
            (t ? ptrB : ptrA)[x] = lo;
            end[x] = base;
            (t ? din : dout)[x] = run;
            if (DIRTY) dirty[x2] = 0;
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(arrive, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    for (int x = threadIdx.x; x < B; x += blockDim.x)
        rcp[x] = 1.0 / ((double)__ldcg(dout + x) + (double)__ldcg(din + x) + (double)B);
    if (threadIdx.x == 0) {
        ptrA[B] = B * B;
        ptrB[B] = B * B;
        *d_nnz = B * B;
        *arrive = 0u;
    }
}

// the dense regime after a MOVE batch whose moves were logged: M and Mt
// updated in place by k_dense_delta, then the line statistics, offsets and
// compaction as in the full path (all three skip when no vertex moved; line
// statistics kept incrementally by returning atomics measured slower: 20K
// round 5 37.7 vs 35.6 us, round 8 33.4 vs 25.6 us)
static void launch_dense_lines(Ctx &c, bool dirty, const int *skip) {
    const int B = c.B;
    const int rg = (int)std::min<long long>(((long long)2 * B + 7) / 8, 148LL * 8);
    if (dirty)
        k_dense_lines<true><<<rg, 256, 0, c.stream>>>(c.dense, c.denseT, B, c.line_dirty, c.bm_rowptr, c.bm_rowend,
                                                      c.bm_col, c.bm_cnt, c.bm_cum, c.bm_colptr, c.bm_colend, c.bm_row,
                                                      c.bm_ccnt, c.bm_ccum, c.dout, c.din, c.rcp, c.d_nnz, c.dl_arrive,
                                                      skip);
    else
        k_dense_lines<false><<<rg, 256, 0, c.stream>>>(c.dense, c.denseT, B, c.line_dirty, c.bm_rowptr, c.bm_rowend,
                                                       c.bm_col, c.bm_cnt, c.bm_cum, c.bm_colptr, c.bm_colend,
                                                       c.bm_row, c.bm_ccnt, c.bm_ccum, c.dout, c.din, c.rcp, c.d_nnz,
                                                       c.dl_arrive, skip);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
}

static void rebuild_dense_delta(Ctx &c) {
    const int B = c.B;
    const int dg = (int)std::min<long long>(((long long)c.delta.count + 7) / 8, 148LL * 8);
    k_dense_delta<<<std::max(dg, 1), 256, 0, c.stream>>>(c.moved, c.moved_cnt, c.delta.first, c.delta.count,
                                                        c.delta.acc, c.oldb, c.b, c.rowptr, c.col, c.wgt, c.cscptr,
                                                        c.cscsrc, c.cscwgt, B, c.dense, c.denseT, c.line_dirty);
    ++c.launches;
    launch_dense_lines(c, true, c.moved_cnt);   // the changed lines only, in place
    c.dense_padded = true;
    c.padded = true;
}

static void rebuild_dense(Ctx &c) {
    nb_join(c);   // k_hist reads the neighbour-block cache
    const int B = c.B, E = c.E;
    const size_t BB = (size_t)B * B;
    GSAP_CUDA(cudaMemsetAsync(c.dense, 0, sizeof(int) * BB, c.stream));
    if (E > 0) {
        int dev_sms = 148;
        if (B <= HIST_SMEM_MAX_B) {
            const size_t smem = sizeof(int) * BB;
            per_device((const void *)k_hist<true>, [] {
                GSAP_CUDA(cudaFuncSetAttribute(k_hist<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                               HIST_SMEM_MAX_B * HIST_SMEM_MAX_B * 4));
                return 1;
            });
            const int grid = (int)std::min<long long>(dev_sms, ((long long)E + 1023) / 1024);
            k_hist<true><<<grid, 1024, smem, c.stream>>>(E, c.esrc, c.nbo, c.wgt, c.b, B, c.dense);
        } else {
            const int grid = (int)std::min<long long>(dev_sms * 8, ((long long)E + 1023) / 1024);
            k_hist<false><<<grid, 1024, 0, c.stream>>>(E, c.esrc, c.nbo, c.wgt, c.b, B, c.dense);
        }
        ++c.launches;
        GSAP_CHECK_LAUNCH();
    }
    dim3 tg((B + 31) / 32, (B + 31) / 32), tb(32, 8);
    k_transpose<<<tg, tb, 0, c.stream>>>(c.dense, B, c.denseT);
    ++c.launches;
    // the lines padded to B entries (a later N2 batch re-compacts only the
    // lines it changed); counts zero beyond each line's end
    GSAP_CUDA(cudaMemsetAsync(c.bm_cnt, 0, sizeof(int) * BB, c.stream));
    GSAP_CUDA(cudaMemsetAsync(c.bm_ccnt, 0, sizeof(int) * BB, c.stream));
    launch_dense_lines(c, false, nullptr);
    c.dense_padded = true;
    c.padded = true;
}

// ---------------------------------------------------------------- sparse --
__global__ void k_rcp(int B, const int *__restrict__ dout, const int *__restrict__ din, double *__restrict__ rcp) {
    for (int x = blockIdx.x * blockDim.x + threadIdx.x; x < B; x += gridDim.x * blockDim.x)
        rcp[x] = 1.0 / ((double)dout[x] + (double)din[x] + (double)B);
}

static void bucket_attrs() {
    per_device((const void *)k_segsort_bucket<1024>, [] {
        GSAP_CUDA(cudaFuncSetAttribute(k_segsort_bucket<1024>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)seg_bucket_smem<1024>()));
        return 1;
    });
}

// the scratch of one side of the multi-kernel sparse rebuild (the two sides
// run concurrently: rows on the context stream, columns on the side stream)
struct LineScratch {
    cudaStream_t st;
    int *len, *cur, *ctr, *nnz, *listW, *listC, *listM, *vpos, *scan_tmp;
    void *seg;
    unsigned long long *xl_keys;
    int *xl_hp;
};

// one side of the sparse blockmodel: lines (rows of M from the out-CSR, or
// columns of M from the in-CSC) by counting sort + per-line segment sort,
// written as a padded CSR: line x's runs stay at its segment offset ptr[x]
// (= the exclusive scan of the line lengths), end[x] marks their end, cnt is
// zero in the rest of the segment.  No second scan and no compaction pass.
template <typename K>
static void build_lines(Ctx &c, const LineScratch &x, const int *gptr, const int *gblk, const int *gw, int *ptr,
                        int *end, int *idx, int *cnt, int *cum, int *deg, int *extent) {
    const cudaStream_t st = x.st;
    Launcher L{st, &c.launches};
    const int B = c.B, V = c.V;
    K *seg = reinterpret_cast<K *>(x.seg);
    GSAP_CUDA(cudaMemsetAsync(x.len, 0, sizeof(int) * (size_t)B, st));
    GSAP_CUDA(cudaMemsetAsync(x.cur, 0, sizeof(int) * (size_t)B, st));
    GSAP_CUDA(cudaMemsetAsync(x.ctr, 0, 8 * sizeof(int), st));
    // each vertex's offset inside its line's segment comes back from the
    // length atomic (vpos), so the scatter has no atomic in its dependent chain
    static const bool no_vpos = getenv("GSAP_SCATTER_ATOMIC") != nullptr;   // A/B switch
    int *vpos = no_vpos ? nullptr : x.vpos;
    k_line_len<<<grid_for(V, 256), 256, 0, st>>>(V, gptr, c.b, x.len, vpos);
    ++c.launches;
    device_scan<int>(x.len, ptr, nullptr, B, false, x.scan_tmp, ptr + B, L);
    k_line_scatter_batched<K><<<grid_for((long long)V, 256), 256, 0, st>>>(V, gptr, gblk, gw, c.b, ptr,
                                                                                x.cur, seg, vpos);
    const LineOut out{cum, end, deg};
    k_line_classify<<<grid_for(B, 256), 256, 0, st>>>(B, ptr, x.nnz, x.listW, x.listC,
                                                           x.ctr, out, extent, SEG_WARP_MAX_MK, x.listM);
    const int gw_ = (int)std::min<long long>(((long long)B + SEG_WARPS - 1) / SEG_WARPS, 148LL * 16);
    per_device((const void *)k_segsort_warp<K, 2>, [] {
        GSAP_CUDA(cudaFuncSetAttribute(k_segsort_warp<K, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)seg_warp2_smem<K>()));
        GSAP_CUDA(cudaFuncSetAttribute(k_segsort_warp<K, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)seg_warp2_smem<K>(512)));
        return 1;
    });
    const int cb = bits_for(B);
    k_segsort_warp<K, 0><<<gw_, SEG_WARPS * 32, 0, st>>>(B, ptr, seg, x.listW, x.ctr, cb, idx, cnt,
                                                              x.nnz, out);
    if (sizeof(K) == 4 && c.prm.line_sort >= 1) {
        // unweighted: one bucket pass + insertion sorts (k_segsort_bucket) for 129..1024 entries
        bucket_attrs();
        const unsigned *useg = reinterpret_cast<const unsigned *>(seg);
        k_segsort_bucket<256><<<gw_, SEG_WARPS * 32, seg_bucket_smem<256>(), st>>>(
            B, ptr, useg, x.listW, 1, x.ctr, 2, cb, idx, cnt, x.nnz, out);
        k_segsort_bucket<512><<<gw_, SEG_WARPS * 32, seg_bucket_smem<512>(), st>>>(
            B, ptr, useg, x.listM, 0, x.ctr, 4, cb, idx, cnt, x.nnz, out);
        k_segsort_bucket<1024><<<gw_, SEG_WARPS * 32, seg_bucket_smem<1024>(), st>>>(
            B, ptr, useg, x.listC, 1, x.ctr, 3, cb, idx, cnt, x.nnz, out);
        c.launches += 4;
    } else {
    k_segsort_warp<K, 1><<<gw_, SEG_WARPS * 32, 0, st>>>(B, ptr, seg, x.listW, x.ctr, cb, idx, cnt,
                                                              x.nnz, out);
    k_segsort_warp<K, 3><<<gw_, SEG_WARPS * 32, seg_warp2_smem<K>(512), st>>>(B, ptr, seg, x.listM,
                                                                                   x.ctr, cb, idx, cnt,
                                                                                   x.nnz, out);
    k_segsort_warp<K, 2><<<gw_, SEG_WARPS * 32, seg_warp2_smem<K>(), st>>>(B, ptr, seg, x.listC,
                                                                                x.ctr, cb, idx, cnt,
                                                                                x.nnz, out);
    c.launches += 4;
    }
    const int gc = (int)std::min<long long>(std::max(1, B / 4), 148LL * 4);
    k_segsort_cta<K><<<gc, 256, 0, st>>>(ptr, seg, x.listC, x.ctr, bits_for(B), idx, cnt,
                                               x.nnz, out);
    k_segsort_xl<K><<<gc, 256, 0, st>>>(ptr, seg, x.listC, x.ctr, bits_for(B), idx, cnt,
                                              x.nnz, reinterpret_cast<K *>(x.xl_keys), x.xl_hp, out);
    c.launches += 5;
    GSAP_CHECK_LAUNCH();
}

// the persistent single-kernel sparse rebuild (coop.cuh)
template <typename K>
static void rebuild_sparse_coop(Ctx &c) {
    const int B = c.B;
    CoopArgs a;
    a.V = c.V;
    a.B = B;
    a.col_bits = bits_for(B);
    a.b = c.b;
    a.kout = c.kout;
    a.kin = c.kin;
    CoopSide &r = a.sd[0], &q = a.sd[1];
    r.gptr = c.rowptr; r.gidx = c.nbo; r.gw = c.wgt;
    r.len = c.seg_len; r.off = c.bm_rowptr; r.cur = c.seg_cur; r.nnz = c.seg_nnz; r.listC = c.seg_listC;
    r.seg = c.keys0; r.tcol = c.bm_col; r.tcnt = c.bm_cnt; r.xl_keys = c.xl_keys; r.xl_hp = c.xl_hp;
    r.cum = c.bm_cum; r.end = c.bm_rowend; r.deg = c.dout;
    q.gptr = c.cscptr; q.gidx = c.nbi; q.gw = c.cscwgt;
    q.len = c.seg2_len; q.off = c.bm_colptr; q.cur = c.seg2_cur; q.nnz = c.seg2_nnz; q.listC = c.seg2_listC;
    q.seg = c.keys1; q.tcol = c.bm_row; q.tcnt = c.bm_ccnt; q.xl_keys = c.xl2_keys; q.xl_hp = c.xl2_hp;
    q.cum = c.bm_ccum; q.end = c.bm_colend; q.deg = c.din;
    a.rcp = c.rcp;
    a.d_nnz = c.d_nnz;
    a.nlong = c.seg_ctr;
    a.bar = c.coop_bar;
    a.moved = nullptr;
    if (c.nb_deferred) {   // the MOVE batch's cache update, in P1
        c.nb_deferred = false;
        a.moved = c.moved; a.moved_cnt = c.moved_cnt; a.movedb = c.movedb;
        a.rowptr = c.rowptr; a.cscptr = c.cscptr; a.csc2csr = c.csc2csr; a.csr2csc = c.csr2csc;
        a.nbo = c.nbo; a.nbi = c.nbi;
    }
    const size_t smem = sizeof(CoopSmem<K>);
    const int grid = per_device((const void *)k_rebuild_coop<K>, [&] {
        GSAP_CUDA(cudaFuncSetAttribute(k_rebuild_coop<K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        int per_sm = 0, sms = 0, dev = 0;
        GSAP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_rebuild_coop<K>, 256, smem));
        GSAP_CUDA(cudaGetDevice(&dev));
        GSAP_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        return std::max(3, per_sm * sms);
    });
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(256);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = c.stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    GSAP_CUDA(cudaLaunchKernelEx(&cfg, k_rebuild_coop<K>, a));
    ++c.launches;
    c.padded = true;
}

static void rebuild_sparse(Ctx &c) {
    const int B = c.B, E = c.E;
    // the scatters read the neighbour-block cache: a side-stream update is
    // joined; a deferred one is done by the persistent kernel's first phase
    nb_join(c, !(E > 0 && c.coop_ok));
    if (E > 0 && c.coop_ok) {
        if (c.weighted) rebuild_sparse_coop<u64>(c);
        else rebuild_sparse_coop<unsigned>(c);
        return;
    }
    if (E == 0) {
        GSAP_CUDA(cudaMemsetAsync(c.bm_rowptr, 0, sizeof(int) * ((size_t)B + 1), c.stream));
        GSAP_CUDA(cudaMemsetAsync(c.bm_colptr, 0, sizeof(int) * ((size_t)B + 1), c.stream));
        GSAP_CUDA(cudaMemsetAsync(c.dout, 0, sizeof(int) * (size_t)B, c.stream));
        GSAP_CUDA(cudaMemsetAsync(c.din, 0, sizeof(int) * (size_t)B, c.stream));
        GSAP_CUDA(cudaMemsetAsync(c.d_nnz, 0, sizeof(int), c.stream));
        return;
    }
    // padded CSR / CSC; d_nnz = the extent E the MDL sums cnt over (zeros in the padding).
    // The two sides are independent: columns on the side stream beside the rows.
    static const bool serial = getenv("GSAP_SIDES_SERIAL") != nullptr;   // A/B switch
    const LineScratch x0{c.stream, c.seg_len, c.seg_cur, c.seg_ctr, c.seg_nnz, c.seg_listW, c.seg_listC,
                         c.seg_listM, c.wa, c.scan_tmp, c.keys0, c.xl_keys, c.xl_hp};
    const LineScratch x1{serial ? c.stream : c.side, c.seg2_len, c.seg2_cur, c.seg2_ctr, c.seg2_nnz, c.seg2_listW,
                         c.seg2_listC, c.seg2_listM, c.wb, c.scan_tmp2, c.keys1, c.xl2_keys, c.xl2_hp};
    if (!serial) {
        GSAP_CUDA(cudaEventRecord(c.ev_rb_fork, c.stream));
        GSAP_CUDA(cudaStreamWaitEvent(c.side, c.ev_rb_fork, 0));
    }
    if (c.weighted) {
        build_lines<u64>(c, x1, c.cscptr, c.nbi, c.cscwgt, c.bm_colptr, c.bm_colend, c.bm_row, c.bm_ccnt, c.bm_ccum,
                         c.din, nullptr);
        build_lines<u64>(c, x0, c.rowptr, c.nbo, c.wgt, c.bm_rowptr, c.bm_rowend, c.bm_col, c.bm_cnt, c.bm_cum,
                         c.dout, c.d_nnz);
    } else {
        build_lines<unsigned>(c, x1, c.cscptr, c.nbi, nullptr, c.bm_colptr, c.bm_colend, c.bm_row, c.bm_ccnt,
                              c.bm_ccum, c.din, nullptr);
        build_lines<unsigned>(c, x0, c.rowptr, c.nbo, nullptr, c.bm_rowptr, c.bm_rowend, c.bm_col, c.bm_cnt,
                              c.bm_cum, c.dout, c.d_nnz);
    }
    if (!serial) {
        GSAP_CUDA(cudaEventRecord(c.ev_rb_join, c.side));
        GSAP_CUDA(cudaStreamWaitEvent(c.stream, c.ev_rb_join, 0));
    }
    c.padded = true;
    GSAP_CHECK_LAUNCH();
}

// export of a padded CSR / CSC line by line: line x's entries [ptr[x],
// end[x]) copied to dst[off[x] ..) (one warp per line, coalesced)
__global__ void k_compact_lines(int B, const int *__restrict__ ptr, const int *__restrict__ end,
                                const int *__restrict__ off, const int *__restrict__ src, int *__restrict__ dst) {
    const int lane = threadIdx.x & 31;
    for (int x = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; x < B; x += (gridDim.x * blockDim.x) >> 5) {
        const int p = ptr[x], n = end[x] - p, o = off[x];
        for (int i = lane; i < n; i += 32) dst[o + i] = src[p + i];
    }
}

void export_lines(Ctx &c, const int *ptr, const int *end, const int *off, const int *src, int *dst) {
    k_compact_lines<<<grid_for(32LL * c.B, 256), 256, 0, c.stream>>>(c.B, ptr, end, off, src, dst);
    ++c.launches;
    GSAP_CHECK_LAUNCH();
}

void rebuild(Ctx &c) {
    nb_refresh(c);   // after a bulk change of b (no-op after a MOVE batch: the apply kept it current)
    cudaEvent_t ev = nullptr;
    kc_begin(c, c.k_rebuild, &ev);
    const bool was_dense = c.dense_mode && c.dense_B == c.B;
    const bool was_padded = c.dense_padded && was_dense;
    c.dense_mode = dense_ok(c, c.B);
    c.padded = false;         // set by the multi-kernel sparse path and the padded dense lines
    c.dense_padded = false;   // set by rebuild_dense (N2 on) and kept by the delta path
    if (c.delta.pending && was_dense && c.dense_mode && c.E > 0 && c.prm.dense_coop && c.B <= SMALL_MAX_B) {
        // N2 at small B: the persistent rebuild (one launch, measured faster than
        // the delta + compaction here), skipped when the batch moved nothing
        launch_rebuild_dense_coop<true>(c, c.moved_cnt);
    } else if (c.delta.pending && was_padded && c.dense_mode && c.E > 0) {
        rebuild_dense_delta(c);   // N2: M, Mt and the padded lines of the previous rebuild + the batch's moves
    } else if (c.dense_mode && c.prm.dense_coop && c.E > 0 && c.B <= SMALL_MAX_B) {
        launch_rebuild_dense_coop<true>(c);
    } else if (c.dense_mode && c.prm.dense_coop == 2 && c.E > 0) {
        launch_rebuild_dense_coop<false>(c);   // measured slower than the multi-kernel path above B = 221
    } else if (c.dense_mode) {
        rebuild_dense(c);   // rcp written by the compaction
    } else {
        rebuild_sparse(c);
        if (!(c.coop_ok && c.E > 0)) {
            k_rcp<<<grid_for(c.B, 256), 256, 0, c.stream>>>(c.B, c.dout, c.din, c.rcp);
            ++c.launches;
        }
    }
    // algorithmic bytes: the compulsory inputs (dst ids,
    // row pointers, b) and the fixed-size outputs (row / column pointers,
    // degrees); the nnz-sized outputs are left out (nnz stays on the device)
    const double bytes = 4.0 * c.E + 8.0 * c.V + 8.0 * (c.B + 1) + 8.0 * c.B;
    c.dense_B = c.dense_mode ? c.B : -1;
    c.delta.pending = false;
    kc_end(c, c.k_rebuild, ev, bytes);
}

}  // namespace gsap
