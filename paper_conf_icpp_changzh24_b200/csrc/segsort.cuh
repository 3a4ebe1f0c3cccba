// segsort.cuh -- the sparse-regime blockmodel rebuild as a counting sort by
// line + per-line sort (Alg. 2, §3.4: "sort_by_key ... segsort ...
// find_subseg_hds ... segreduce"), without a global sort of 64-bit keys:
//
//   1. line lengths: len[b[v]] += deg(v)                  (one atomic per vertex)
//   2. offsets: exclusive scan of len
//   3. scatter: each vertex appends the blocks of its neighbours to its line's
//      segment (one atomic per vertex, 32 vertices per warp step; the order
//      inside a segment is arbitrary, the sort below makes it canonical)
//   4. per segment: sort + run-length encode (a warp for <= 512 entries, a CTA
//      in shared memory for <= 4096, a CTA in global scratch beyond); the runs
//      stay at the segment offset (padded CSR: end[x], cum, line sums and
//      zero counts in the padding written by the same warp / CTA), or go to
//      scratch for the persistent kernel's compaction (coop.cuh).
//
// Keys are the neighbour block (unweighted, u32) or (block << 32 | weight)
// (weighted, u64): equal blocks become adjacent and their weights are summed.
#pragma once

#include "common.cuh"

namespace gsap {

constexpr int SEG_WARP_MAX = 512;    // entries sorted by one warp in shared memory
constexpr int SEG_WARPS = 8;

// entries one CTA sorts in shared memory (48 KB of static shared memory)
template <typename K>
struct SegCta {
    static constexpr int CAP = sizeof(K) == 8 ? 2048 : 4096;
};

template <typename K>
GSAP_DEV int key_col(K k) { return sizeof(K) == 8 ? (int)(k >> 32) : (int)k; }
template <typename K>
GSAP_DEV int key_w(K k) { return sizeof(K) == 8 ? (int)(unsigned)(k & 0xffffffffULL) : 1; }
template <typename K>
GSAP_DEV K key_max() { return (K)~(K)0; }

template <int NT>
GSAP_DEV void nt_sync() {
    if (NT == 32) __syncwarp();
    else __syncthreads();
}

// bitonic sort of a[0, n), n a power of two, by NT cooperating threads
template <typename K, int NT>
GSAP_DEV void bitonic(K *a, int n, int tid) {
    for (int k = 2; k <= n; k <<= 1) {
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = tid; i < (n >> 1); i += NT) {
                const int lo = ((i & ~(j - 1)) << 1) | (i & (j - 1));
                const int hi = lo + j;
                const bool up = (lo & k) == 0;
                const K x = a[lo], y = a[hi];
                if ((x > y) == up) {
                    a[lo] = y;
                    a[hi] = x;
                }
            }
            nt_sync<NT>();
        }
    }
}

// run-length encode sorted a[0, L) by NT threads: hp[q] = start of run q;
// writes (block, summed weight) of run q to ocol/ocnt[q]; returns the run count
template <typename K, int NT>
GSAP_DEV int rle_runs(const K *a, int L, int *hp, int *ocol, int *ocnt, int tid, int *sh) {
    // each thread takes a contiguous chunk so the runs come out in order
    const int chunk = (L + NT - 1) / NT;
    const int lo = min(L, tid * chunk), hi = min(L, lo + chunk);
    int heads = 0;
    for (int i = lo; i < hi; ++i) heads += (i == 0 || key_col(a[i]) != key_col(a[i - 1])) ? 1 : 0;
    // exclusive scan of heads over the NT threads
    int x = heads;
    const int lane = tid & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += t;
    }
    int base = x - heads, total;
    if (NT == 32) {
        total = __shfl_sync(FULL, x, 31);
    } else {
        const int w = tid >> 5;
        if (lane == 31) sh[w] = x;
        __syncthreads();
        int wb = 0;
        total = 0;
        for (int i = 0; i < NT / 32; ++i) {
            if (i < w) wb += sh[i];
            total += sh[i];
        }
        base += wb;
        __syncthreads();
    }
    for (int i = lo; i < hi; ++i)
        if (i == 0 || key_col(a[i]) != key_col(a[i - 1])) hp[base++] = i;
    nt_sync<NT>();
    for (int q = tid; q < total; q += NT) {
        const int s = hp[q], e = q + 1 < total ? hp[q + 1] : L;
        int c;
        if (sizeof(K) == 8) {
            c = 0;
            for (int i = s; i < e; ++i) c += key_w(a[i]);
        } else {
            c = e - s;
        }
        ocol[q] = key_col(a[s]);
        ocnt[q] = c;
    }
    nt_sync<NT>();
    return total;
}

// padded output (rebuild_sparse, multi-kernel): the runs of line x stay at
// its segment offset o in the final idx / cnt arrays; the epilogue writes the
// in-line prefix cum, zeroes cnt in the padding [o + u, o + L), and records
// end[x] = o + u and the line's total weight deg[x].  cum == nullptr: off.
struct LineOut {
    int *cum, *end, *deg;
};

template <int NT>
GSAP_DEV void line_epilogue(const LineOut &out, int *__restrict__ cnt, int o, int u, int L, int x, int tid,
                            int *sh) {
    nt_sync<NT>();   // the runs written by the other threads are visible
    const int lane = tid & 31, w = tid >> 5;
    int carry = 0;
    for (int base = 0; base < u; base += NT) {
        const int i = base + tid;
        const int c = i < u ? cnt[o + i] : 0;
        const int xi = warp_incl_scan(c);
        int before = 0, total;
        if (NT == 32) {
            total = __shfl_sync(FULL, xi, 31);
        } else {
            if (lane == 31) sh[w] = xi;
            __syncthreads();
            total = 0;
            for (int q = 0; q < NT / 32; ++q) {
                const int t = sh[q];
                if (q < w) before += t;
                total += t;
            }
            __syncthreads();
        }
        if (i < u) out.cum[o + i] = carry + before + xi;
        carry += total;
    }
    for (int i = u + tid; i < L; i += NT) cnt[o + i] = 0;
    if (tid == 0) {
        out.end[x] = o + u;
        out.deg[x] = carry;
    }
}

// 1. len[b[v]] += deg(v); with vpos: the returned old length is v's offset
// inside its line's segment (vpos[v]), so the scatter places v's entries
// without an atomic of its own (multi-kernel path)
__global__ void k_line_len(int V, const int *__restrict__ gptr, const int *__restrict__ b, int *__restrict__ len,
                           int *__restrict__ vpos) {
    for (int v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) {
        const int d = gptr[v + 1] - gptr[v];
        if (vpos) vpos[v] = d ? atomicAdd(len + b[v], d) : 0;
        else if (d) atomicAdd(len + b[v], d);
    }
}

// 3'. the scatter as warp-batched tasks (task = (side, vertex), sides 0..nsides-1
// of V vertices each): lane l claims task (base + l)'s slot range with one
// atomic -- 32 claims in flight instead of one per warp step -- then the warp
// copies the 32 tasks' entries flattened (lane-parallel over the batch's
// entries, owner task found by a 5-step search over the lanes' offsets), so
// every lane has an independent gather in flight.
template <typename K>
struct ScatterSide {
    const int *__restrict__ gptr;
    const int *__restrict__ gblk;   // the neighbours' blocks, parallel to the adjacency (nbo / nbi)
    const int *__restrict__ gw;
    const int *off;   // written earlier in the same kernel (coop): plain loads
    int *cur;
    K *seg;
    const int *vpos;  // nullptr: claim each vertex's slots with an atomic on cur; else vpos[v] (k_line_len)
};

template <typename K>
GSAP_DEV void scatter_batched(const ScatterSide<K> &s0, const ScatterSide<K> &s1, int nsides, int V,
                              const int *__restrict__ b, int gwarp, int gwarps) {
    const int lane = threadIdx.x & 31;
    const int ntasks = nsides * V;
    for (int base = gwarp * 32; base < ntasks; base += gwarps * 32) {
        const int task = base + lane;
        int q = 0, lo = 0, n = 0, pos = 0;
        if (task < ntasks) {
            q = task >= V;
            const int v = q ? task - V : task;
            const int *gptr = q ? s1.gptr : s0.gptr;
            lo = __ldg(gptr + v);
            n = __ldg(gptr + v + 1) - lo;
            if (n) {
                const int x = __ldg(b + v);
                const ScatterSide<K> &sd = q ? s1 : s0;
                pos = sd.off[x] + (sd.vpos ? __ldg(sd.vpos + v) : atomicAdd(sd.cur + x, n));
            }
        }
        const int incl = warp_incl_scan(n);
        const int total = __shfl_sync(FULL, incl, 31);
        const int excl = incl - n;
        constexpr int U = 4;   // entries per lane per step: U independent gathers in flight
        for (int f0 = 0; f0 < total; f0 += 32 * U) {
            int src[U], dst[U], wq[U], nbr[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int f = f0 + u * 32 + lane;
                int t = 0;   // the last lane whose offset is <= f owns entry f
#pragma unroll
                for (int step = 16; step >= 1; step >>= 1) {
                    const int cand = t + step;
                    const int ex = __shfl_sync(FULL, excl, cand & 31);
                    if (cand < 32 && ex <= f) t = cand;
                }
                const int tq = __shfl_sync(FULL, q, t), tlo = __shfl_sync(FULL, lo, t);
                const int tpos = __shfl_sync(FULL, pos, t), tex = __shfl_sync(FULL, excl, t);
                wq[u] = f < total ? tq : -1;
                src[u] = tlo + f - tex;
                dst[u] = tpos + f - tex;
            }
#pragma unroll
            for (int u = 0; u < U; ++u) nbr[u] = wq[u] >= 0 ? __ldg((wq[u] ? s1.gblk : s0.gblk) + src[u]) : 0;
            int blk[U], wt[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                blk[u] = nbr[u];   // the neighbour-block cache: no gather of b
                wt[u] = (sizeof(K) == 8 && wq[u] >= 0) ? __ldg((wq[u] ? s1.gw : s0.gw) + src[u]) : 0;
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (wq[u] < 0) continue;
                K *seg = wq[u] ? s1.seg : s0.seg;
                if (sizeof(K) == 8) seg[dst[u]] = (K)(((unsigned long long)(unsigned)blk[u] << 32) | (unsigned)wt[u]);
                else seg[dst[u]] = (K)(unsigned)blk[u];
            }
        }
    }
}

template <typename K>
__global__ void k_line_scatter_batched(int V, const int *__restrict__ gptr, const int *__restrict__ gblk,
                                       const int *__restrict__ gw, const int *__restrict__ b,
                                       const int *__restrict__ off, int *__restrict__ cur, K *__restrict__ seg,
                                       const int *__restrict__ vpos) {
    const ScatterSide<K> sd{gptr, gblk, gw, off, cur, seg, vpos};
    scatter_batched<K>(sd, sd, 1, V, b, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, (gridDim.x * blockDim.x) >> 5);
}

// 4a. classify lines by segment length
__global__ void k_line_classify(int B, const int *__restrict__ off, int *__restrict__ nnz, int *__restrict__ listW,
                                int *__restrict__ listC, int *__restrict__ counters, LineOut out,
                                int *__restrict__ extent, int warp_max, int *__restrict__ listM) {
    if (extent && blockIdx.x == 0 && threadIdx.x == 0) *extent = off[B];
    for (int x = blockIdx.x * blockDim.x + threadIdx.x; x < B; x += gridDim.x * blockDim.x) {
        const int L = off[x + 1] - off[x];
        if (L == 0) {
            nnz[x] = 0;
            if (out.cum) {
                out.end[x] = off[x];
                out.deg[x] = 0;
            }
        }
        else if (L <= 128) listW[atomicAdd(counters, 1)] = x;                           // warp mode 0
        else if (L <= 256) listW[B - 1 - atomicAdd(counters + 2, 1)] = x;               // warp mode 1
        else if (listM && L <= 512) listM[atomicAdd(counters + 4, 1)] = x;              // warp mode 3
        else if (L <= warp_max) listC[B - 1 - atomicAdd(counters + 3, 1)] = x;          // warp mode 2
        else listC[atomicAdd(counters + 1, 1)] = x;                                      // CTA
    }
}

// bitonic sort of 32*E keys held in registers, blocked layout (lane l holds
// elements l*E .. l*E+E-1): partners inside a lane swap registers, partners
// in other lanes come over __shfl_xor_sync.  Fully unrolled.
template <typename K, int E>
GSAP_DEV void warp_bitonic(K (&v)[E]) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int k = 2; k <= 32 * E; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            if (j >= E) {
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    const int i = lane * E + e;
                    const K o = __shfl_xor_sync(FULL, v[e], j / E);
                    const bool up = (i & k) == 0, lower = (i & j) == 0;
                    v[e] = (lower == up) ? (v[e] < o ? v[e] : o) : (v[e] < o ? o : v[e]);
                }
            } else {
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    if ((e & j) == 0) {
                        const int i = lane * E + e;
                        const bool up = (i & k) == 0;
                        const K a = v[e], b = v[e + j];
                        if ((a > b) == up) {
                            v[e] = b;
                            v[e + j] = a;
                        }
                    }
                }
            }
        }
    }
}

// sort + RLE of one segment of L <= 32*E keys by one warp, in registers;
// runs written to ocol / ocnt, returns the run count (warp-uniform)
template <typename K, int E>
GSAP_DEV int warp_segsort_rle(const K *__restrict__ src, int L, int *__restrict__ ocol, int *__restrict__ ocnt) {
    const int lane = threadIdx.x & 31;
    K v[E];
#pragma unroll
    for (int e = 0; e < E; ++e) {   // coalesced (striped) load: the sort permutes anyway
        const int i = e * 32 + lane;
        v[e] = i < L ? src[i] : key_max<K>();
    }
    warp_bitonic<K, E>(v);
    // run heads and their ranks
    const K prev_last = __shfl_up_sync(FULL, v[E - 1], 1);
    int heads = 0;
    bool head[E];
#pragma unroll
    for (int e = 0; e < E; ++e) {
        const int i = lane * E + e;
        const K p = e == 0 ? prev_last : v[e - 1];
        head[e] = i < L && (i == 0 || key_col(v[e]) != key_col(p));
        heads += head[e] ? 1 : 0;
    }
    int x = heads;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += t;
    }
    const int total = __shfl_sync(FULL, x, 31);
    int q = x - heads;
    // weight of each run: inclusive prefix of weights, differenced at heads
    int wsum[E], run = 0;
#pragma unroll
    for (int e = 0; e < E; ++e) {
        const int i = lane * E + e;
        run += i < L ? key_w(v[e]) : 0;
        wsum[e] = run;
    }
    int y = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(FULL, y, o);
        if (lane >= o) y += t;
    }
    const int lane_base = y - run;   // weight before this lane's first element
    // a run's weight = (prefix at its last element) - (prefix before its head):
    // the head's lane writes the negative start prefix, then (after a
    // __syncwarp) the lane holding the run's last element adds its prefix
#pragma unroll
    for (int e = 0; e < E; ++e) {
        if (head[e]) {
            ocol[q] = key_col(v[e]);
            ocnt[q] = -(lane_base + (e == 0 ? 0 : wsum[e - 1]));
            ++q;
        }
    }
    __syncwarp();
    const bool nb_head0 = __shfl_down_sync(FULL, head[0] ? 1 : 0, 1) != 0;   // lane+1's first flag
    const int qbase = x - heads;
    int seen = 0;
#pragma unroll
    for (int e = 0; e < E; ++e) {
        const int i = lane * E + e;
        seen += head[e] ? 1 : 0;
        if (i < L && (i == L - 1 || (e + 1 < E ? head[e + 1] : nb_head0)))
            ocnt[qbase + seen - 1] += lane_base + wsum[e];
    }
    __syncwarp();
    return total;
}

// 4b. warp-sized segments: one warp each, three instantiations, each over its
// own line list (k_line_classify), so that a heavy path does not lower the
// occupancy of the common one:
//   MODE 0: <= 128 entries, bitonic + RLE in registers;
//   MODE 1: 129..256 entries in registers (8 per lane);
//   MODE 3: 257..512 entries, the MODE 2 sort with half-size buffers (own
//           list: more CTAs per SM for the shorter lines);
//   MODE 2: 257 (513 with MODE 3)..SEG_WARP_MAX_MK entries: the stable LSD radix sort over the
//           key's block bits (cta_radix_sort with 32 threads: 4-bit digits,
//           per-lane packed counters, no atomics; O(L) per pass instead of
//           bitonic's O(L log^2 L)) in dynamic shared memory, then RLE.
#ifndef GSAP_SEG_WARP_MAX_MK
#define GSAP_SEG_WARP_MAX_MK 1024
#endif
constexpr int SEG_WARP_MAX_MK = GSAP_SEG_WARP_MAX_MK;   // multi-kernel path: longer lines go to the CTA sorts
template <typename K>
constexpr size_t seg_warp2_smem(int cap = SEG_WARP_MAX_MK) {
    return (size_t)SEG_WARPS * (2 * (size_t)cap * sizeof(K) + 8 * 32 * sizeof(unsigned));
}

template <typename K, int NT>
GSAP_DEV K *cta_radix_sort(K *a, K *b, int L, int col_bits, unsigned *cntp, unsigned *wsum);

template <typename K, int MODE>
__global__ void __launch_bounds__(SEG_WARPS * 32) k_segsort_warp(int B, const int *__restrict__ off, K *__restrict__ seg,
                                                                 const int *__restrict__ listW,
                                                                 const int *__restrict__ counters, int col_bits,
                                                                 int *__restrict__ tcol, int *__restrict__ tcnt,
                                                                 int *__restrict__ nnz, LineOut out) {
    extern __shared__ __align__(16) unsigned char seg_dyn[];   // MODE 2/3: SEG_WARPS x (2 key buffers) + counters
    constexpr int CAP = MODE == 3 ? 512 : SEG_WARP_MAX_MK;     // key buffer per warp (MODE 2 / 3)
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int n_lines = counters[MODE == 0 ? 0 : MODE == 1 ? 2 : MODE == 2 ? 3 : 4];
    for (int li = blockIdx.x * SEG_WARPS + w; li < n_lines; li += gridDim.x * SEG_WARPS) {
        // MODE 2: listW is the CTA list (listC), filled from its back; MODE 3: listM, from its front
        const int x = (MODE == 0 || MODE == 3) ? listW[li] : listW[B - 1 - li];
        const int o = off[x], L = off[x + 1] - o;
        int u;
        if (MODE == 1) {
            u = warp_segsort_rle<K, 8>(seg + o, L, tcol + o, tcnt + o);
        } else if (MODE == 0) {
            if (L <= 32) u = warp_segsort_rle<K, 1>(seg + o, L, tcol + o, tcnt + o);
            else if (L <= 64) u = warp_segsort_rle<K, 2>(seg + o, L, tcol + o, tcnt + o);
            else u = warp_segsort_rle<K, 4>(seg + o, L, tcol + o, tcnt + o);
        } else {
            K *ka = reinterpret_cast<K *>(seg_dyn) + (size_t)w * 2 * CAP;
            K *kb = ka + CAP;
            unsigned *cntp = reinterpret_cast<unsigned *>(reinterpret_cast<K *>(seg_dyn) +
                                                          (size_t)SEG_WARPS * 2 * CAP) + w * 8 * 32;
            for (int i = lane; i < L; i += 32) ka[i] = seg[o + i];
            __syncwarp();
            K *keys = cta_radix_sort<K, 32>(ka, kb, L, col_bits, cntp, nullptr);
            int *hw = reinterpret_cast<int *>(keys == ka ? kb : ka);
            u = rle_runs<K, 32>(keys, L, hw, tcol + o, tcnt + o, lane, nullptr);
        }
        if (lane == 0) nnz[x] = u;
        if (out.cum) line_epilogue<32>(out, tcnt, o, u, L, x, lane, nullptr);
    }
}

// 4b'. unweighted graphs (32-bit keys = the neighbour block): 129..CAP-entry
// segments, one warp each, sorted by ONE MSD bucket pass + an insertion sort
// inside each bucket (O(L) expected work, against bitonic's O(L log^2 L) or
// the radix sort's ceil(col_bits / 4) passes): the keys stay in registers
// (striped), nb = pow2 >= L buckets over the line's key range [mn, mx] by the
// monotone map floor((k - mn) nb / (mx - mn + 1)) in fp32 (monotone: every
// step rounds monotonically), bucket counts by shared-memory atomics, one
// warp scan, scatter to bucket start + the key's rank from the counting atomic
// (order inside a bucket arbitrary), then each lane insertion-sorts the range
// of its buckets.  A line whose fullest bucket
// holds > 64 keys (clustered ids) takes the 4-bit radix sort instead.  The
// RLE is a ballot over the sorted keys; with unit weights a run's count is
// the distance between heads and cum is the run's end position, so the
// padded CSR epilogue needs no scan.  Same output as k_segsort_warp.
constexpr int SEG_BUCKET_FALLBACK = 64;
template <int CAP>
constexpr size_t seg_bucket_smem() {
    return (size_t)SEG_WARPS * (2 * (size_t)CAP * sizeof(unsigned) + 8 * 32 * sizeof(unsigned));
}

template <typename K, int NT>
GSAP_DEV K *cta_radix_sort(K *a, K *b, int L, int col_bits, unsigned *cntp, unsigned *wsum);

// one line seg[0, L) (32-bit keys, 129 <= L <= CAP) by one warp: sorted,
// run-length encoded and written in the padded CSR layout at line offset 0 of
// tcol / tcnt / cum (the padding's counts zeroed); kb, cb: CAP words of the
// warp's shared memory each, cntp: 256 words (radix fallback).  Returns the
// run count.  Warp-uniform.
template <int CAP>
GSAP_DEV int warp_bucket_line(const unsigned *__restrict__ seg, int L, int col_bits, unsigned *kb, int *cb,
                              unsigned *cntp, int *__restrict__ tcol, int *__restrict__ tcnt, int *__restrict__ cum) {
    constexpr int E = CAP / 32;
    const int lane = threadIdx.x & 31;
    const unsigned lt = (1u << lane) - 1u;
    unsigned k[E];
    unsigned mn = 0xffffffffu, mx = 0u;
#pragma unroll
    for (int e = 0; e < E; ++e) {
        const int i = e * 32 + lane;
        k[e] = i < L ? seg[i] : 0u;
        if (i < L) {
            mn = min(mn, k[e]);
            mx = max(mx, k[e]);
        }
    }
    mn = __reduce_min_sync(FULL, mn);
    mx = __reduce_max_sync(FULL, mx);
    int lp = 0;
    while ((32 << lp) < L) ++lp;   // nb = 32 << lp buckets, warp-uniform, <= CAP
    const int nb = 32 << lp, per = 1 << lp;
    const float scale = (float)nb / ((float)(mx - mn) + 1.0f);
    // bucket q lives at slot (q mod per) * 32 + q / per: lane l owns the
    // consecutive buckets l per .. l per + per - 1 for the scan, and the
    // scan's accesses (all lanes at the same j) hit 32 distinct banks
    auto slot = [&](unsigned key) {
        const int q = min(nb - 1, (int)((float)(key - mn) * scale));
        return ((q & (per - 1)) << 5) | (q >> lp);
    };
    for (int j = lane; j < nb; j += 32) cb[j] = 0;
    __syncwarp();
    // counts; the returned old count is the key's rank inside its bucket, so
    // the scatter below needs no atomic.  CAP <= 512: (slot << 16 | rank) kept
    // per key; CAP 1024 (register budget): two 16-bit ranks per register, the
    // slot recomputed
#ifndef GSAP_BUCKET_PACK
#define GSAP_BUCKET_PACK 1
#endif
    constexpr bool PACK = GSAP_BUCKET_PACK && CAP <= 512;
    constexpr int NR = PACK ? E : (E + 1) / 2;
    unsigned rk[NR];
#pragma unroll
    for (int e = 0; e < NR; ++e) rk[e] = 0u;
#pragma unroll
    for (int e = 0; e < E; ++e) {
        if (e * 32 + lane < L) {
            const int sl = slot(k[e]);
            const unsigned rank = (unsigned)atomicAdd(&cb[sl], 1);
            if (PACK) rk[e] = ((unsigned)sl << 16) | rank;
            else rk[e >> 1] |= rank << ((e & 1) * 16);
        }
    }
    __syncwarp();
    // exclusive scan of the buckets in order
    int tot = 0, mxc = 0;
    for (int j = 0; j < per; ++j) {
        const int cj = cb[(j << 5) | lane];
        tot += cj;
        mxc = max(mxc, cj);
    }
    int run = warp_incl_scan(tot) - tot;
    for (int j = 0; j < per; ++j) {
        const int cj = cb[(j << 5) | lane];
        cb[(j << 5) | lane] = run;
        run += cj;
    }
    const int fullest = __reduce_max_sync(FULL, mxc);
    __syncwarp();
    unsigned *sorted = kb;
    int *hp = cb;
    if (fullest > SEG_BUCKET_FALLBACK && mn != mx) {
#pragma unroll
        for (int e = 0; e < E; ++e)
            if (e * 32 + lane < L) kb[e * 32 + lane] = k[e];
        __syncwarp();
        sorted = cta_radix_sort<unsigned, 32>(kb, reinterpret_cast<unsigned *>(cb), L, col_bits, cntp, nullptr);
        hp = reinterpret_cast<int *>(sorted == kb ? reinterpret_cast<unsigned *>(cb) : kb);
    } else {
#pragma unroll
        for (int e = 0; e < E; ++e) {
            if (e * 32 + lane < L) {
                if (PACK) kb[cb[rk[e] >> 16] + (rk[e] & 0xffffu)] = k[e];
                else kb[cb[slot(k[e])] + ((rk[e >> 1] >> ((e & 1) * 16)) & 0xffffu)] = k[e];
            }
        }
        // lane l's buckets l per .. l per + per - 1 are the contiguous range
        // [start of bucket l per, start of bucket (l + 1) per) = [cb[l], cb[l + 1])
        const int s0 = cb[lane], e0 = lane < 31 ? cb[lane + 1] : L;
        __syncwarp();
        // one insertion sort over the lane's whole range: the buckets are
        // already in order, so keys only move inside their bucket (cost =
        // range + inversions; no per-bucket loop, little divergence)
        // (the sorted prefix's maximum is carried in a register: a key not below
        // it -- the common case -- costs one load and no store)
        unsigned mxk = s0 < e0 ? kb[s0] : 0u;
        for (int i = s0 + 1; i < e0; ++i) {
            const unsigned key = kb[i];
            if (key >= mxk) {
                mxk = key;
                continue;
            }
            int q = i - 1;
            unsigned prev = mxk;
            while (prev > key) {
                kb[q + 1] = prev;
                if (--q < s0) break;
                prev = kb[q];
            }
            kb[q + 1] = key;
        }
        __syncwarp();
    }
#ifndef GSAP_BUCKET_FUSED_RLE
#define GSAP_BUCKET_FUSED_RLE 0   // measured slower (2M rebuild r4 / r6 1.46 / 1.28 vs 1.40 / 1.19 ms)
#endif
#if !GSAP_BUCKET_FUSED_RLE
    // run heads (ballot), then per run: block, count, cum = end position
    int u = 0;
    unsigned carry = 0u;   // the previous chunk's last key (lane 31)
    for (int base = 0; base < L; base += 32) {
        const int i = base + lane;
        const unsigned k0 = i < L ? sorted[i] : 0u;
        unsigned kp = __shfl_up_sync(FULL, k0, 1);
        if (lane == 0) kp = carry;
        const bool head = i < L && (i == 0 || k0 != kp);
        const unsigned bal = __ballot_sync(FULL, head);
        if (head) hp[u + __popc(bal & lt)] = i;
        u += __popc(bal);
        carry = __shfl_sync(FULL, k0, 31);
    }
    __syncwarp();
    for (int q = lane; q < u; q += 32) {
        const int s0 = hp[q], e0 = q + 1 < u ? hp[q + 1] : L;
        tcol[q] = (int)sorted[s0];
        tcnt[q] = e0 - s0;
        cum[q] = e0;
    }
#else
    // runs, one 32-key chunk at a time with the next chunk's head ballot in
    // hand: a head's run ends at the next head (later in its chunk, else the
    // first head of the next chunk; a run spanning a whole chunk is scanned
    // for by its lane); per run: block, count, cum = end position (written
    // directly, consecutive runs to consecutive q)
    (void)hp;
    unsigned kc = 0u, hc = 0u;
    {
        const bool h = lane < L && (lane == 0 || sorted[lane] != sorted[lane - 1]);
        kc = lane < L ? sorted[lane] : 0u;
        hc = __ballot_sync(FULL, h);
    }
    int u = 0;
    for (int base = 0; base < L; base += 32) {
        const int i = base + lane, in = i + 32;
        const bool hn_ = in < L && sorted[in] != sorted[in - 1];
        const unsigned kn = in < L ? sorted[in] : 0u;
        const unsigned hn = __ballot_sync(FULL, hn_);
        if ((hc >> lane) & 1u) {
            const unsigned later = hc & ~((2u << lane) - 1u);   // heads after this lane in the chunk
            int e;
            if (later) e = base + __ffs(later) - 1;
            else if (hn) e = base + 32 + __ffs(hn) - 1;
            else {   // no head in the next chunk: the run spans it (or the line ends)
                e = min(L, base + 64);
                while (e < L && sorted[e] == kc) ++e;
            }
            const int q = u + __popc(hc & lt);
            tcol[q] = (int)kc;
            tcnt[q] = e - i;
            cum[q] = e;
        }
        u += __popc(hc);
        hc = hn;
        kc = kn;
    }
#endif
    for (int i = u + lane; i < L; i += 32) tcnt[i] = 0;
    __syncwarp();   // the buffers are reused by the next line
    return u;
}

template <int CAP>
__global__ void __launch_bounds__(SEG_WARPS * 32, CAP >= 512 ? 3 : 1) k_segsort_bucket(int B, const int *__restrict__ off,
                                                                   const unsigned *__restrict__ seg,
                                                                   const int *__restrict__ list, int from_back,
                                                                   const int *__restrict__ counters, int ctr,
                                                                   int col_bits, int *__restrict__ tcol,
                                                                   int *__restrict__ tcnt, int *__restrict__ nnz,
                                                                   LineOut out) {
    extern __shared__ __align__(16) unsigned char seg_dyn[];
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned *kb = reinterpret_cast<unsigned *>(seg_dyn) + (size_t)w * (2 * CAP + 256);
    int *cb = reinterpret_cast<int *>(kb + CAP);        // bucket counts -> cursors -> run heads
    unsigned *cntp = kb + 2 * CAP;                      // radix fallback counters (8 x 32)
    const int n_lines = counters[ctr];
    for (int li = blockIdx.x * SEG_WARPS + w; li < n_lines; li += gridDim.x * SEG_WARPS) {
        const int x = from_back ? list[B - 1 - li] : list[li];
        const int o = off[x], L = off[x + 1] - o;
        const int u = warp_bucket_line<CAP>(seg + o, L, col_bits, kb, cb, cntp, tcol + o, tcnt + o, out.cum + o);
        if (lane == 0) {
            nnz[x] = u;
            out.end[x] = o + u;
            out.deg[x] = L;
        }
    }
}

// stable LSD radix sort of a[0, L) by the block bits of the key (key_col),
// 4-bit digits, NT threads.  Each thread owns a contiguous chunk of an odd
// number of keys (conflict-free shared-memory strides); its 16 digit
// counters are packed two per word (16-bit fields, L <= 4096) in its own
// column of cntp[8][NT], so counting needs no atomics, and one block-wide
// scan of the packed 8-word vectors gives every (digit, thread) offset.
// Ping-pongs between a and b; returns the buffer holding the result.
// O(L * passes) instead of bitonic's O(L log^2 L).
template <typename K, int NT>
GSAP_DEV K *cta_radix_sort(K *a, K *b, int L, int col_bits, unsigned *cntp, unsigned *wsum) {
    const int tid = threadIdx.x % NT, lane = tid & 31, w = tid >> 5;
    const int C = ((L + NT - 1) / NT) | 1;
    const int lo = min(L, tid * C), hi = min(L, lo + C);
    for (int sh = 0; sh < col_bits; sh += 4) {
#pragma unroll
        for (int k = 0; k < 8; ++k) cntp[k * NT + tid] = 0u;
        for (int i = lo; i < hi; ++i) {
            const int d = (key_col(a[i]) >> sh) & 15;
            cntp[(d >> 1) * NT + tid] += 1u << ((d & 1) * 16);
        }
        unsigned c[8], x[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) x[k] = c[k] = cntp[k * NT + tid];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                const unsigned t = __shfl_up_sync(FULL, x[k], o);
                if (lane >= o) x[k] += t;
            }
        }
        if (NT > 32) {
            if (lane == 31) {
#pragma unroll
                for (int k = 0; k < 8; ++k) wsum[w * 8 + k] = x[k];
            }
            __syncthreads();
        }
        unsigned wp[8], tot[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            wp[k] = 0u;
            tot[k] = NT > 32 ? 0u : __shfl_sync(FULL, x[k], 31);
        }
        if (NT > 32) {
            for (int q = 0; q < NT / 32; ++q) {
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const unsigned v = wsum[q * 8 + k];
                    wp[k] += q < w ? v : 0u;
                    tot[k] += v;
                }
            }
        }
        unsigned run = 0u;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const unsigned t0 = tot[k] & 0xffffu, t1 = tot[k] >> 16;
            const unsigned base = run | ((run + t0) << 16);   // bases of digits 2k, 2k + 1
            run += t0 + t1;
            cntp[k * NT + tid] = x[k] - c[k] + wp[k] + base;
        }
        for (int i = lo; i < hi; ++i) {
            const K key = a[i];
            const int d = (key_col(key) >> sh) & 15;
            const unsigned f = (d & 1) * 16;
            const unsigned p = cntp[(d >> 1) * NT + tid];
            cntp[(d >> 1) * NT + tid] = p + (1u << f);
            b[(p >> f) & 0xffffu] = key;
        }
        nt_sync<NT>();
        K *t = a;
        a = b;
        b = t;
    }
    return a;
}

#ifndef GSAP_CTA_BITONIC_MAX
#define GSAP_CTA_BITONIC_MAX 0   // > 0: CTA bitonic up to this length (measured slower than the radix
                                 // sort on B200: 20K 126 vs 97 us, 200K 408 vs 334 us per rebuild)
#endif
// one line of L <= SegCta::CAP keys sorted by a 256-thread CTA in shared
// memory: the 4-bit LSD radix sort (or bitonic up to GSAP_CTA_BITONIC_MAX).
// Returns the buffer holding the sorted keys (the other one is free).
template <typename K>
GSAP_DEV K *cta_sort(const K *__restrict__ src, int L, K *a, K *b, int col_bits, unsigned *cntp, unsigned *wsum) {
    if (L <= GSAP_CTA_BITONIC_MAX) {
        int n = 1;
        while (n < L) n <<= 1;
        for (int i = threadIdx.x; i < n; i += 256) a[i] = i < L ? src[i] : key_max<K>();
        __syncthreads();
        bitonic<K, 256>(a, n, threadIdx.x);
        return a;
    }
    for (int i = threadIdx.x; i < L; i += 256) a[i] = src[i];
    __syncthreads();
    return cta_radix_sort<K, 256>(a, b, L, col_bits, cntp, wsum);
}

// 4c. long segments: one CTA each, in shared memory (<= 4096) or in a global
// scratch region at 2 * off (Sum of regions <= 2E)
template <typename K>
__global__ void __launch_bounds__(256) k_segsort_cta(const int *__restrict__ off, K *__restrict__ seg,
                                                     const int *__restrict__ listC, const int *__restrict__ counters,
                                                     int col_bits, int *__restrict__ tcol, int *__restrict__ tcnt,
                                                     int *__restrict__ nnz, LineOut out) {
    constexpr int CAP = SegCta<K>::CAP;
    __shared__ K skeys[2][CAP];
    __shared__ unsigned cntp[8 * 256];
    __shared__ unsigned wsum[8 * 8];
    __shared__ int sh[8];
    const int n_lines = counters[1];
    for (int li = blockIdx.x; li < n_lines; li += gridDim.x) {
        const int x = listC[li];
        const int o = off[x], L = off[x + 1] - o;
        if (L > CAP) continue;   // k_segsort_xl
        K *keys = cta_sort(seg + o, L, skeys[0], skeys[1], col_bits, cntp, wsum);
        int *hp = reinterpret_cast<int *>(keys == skeys[0] ? skeys[1] : skeys[0]);
        const int u = rle_runs<K, 256>(keys, L, hp, tcol + o, tcnt + o, threadIdx.x, sh);
        if (threadIdx.x == 0) nnz[x] = u;
        if (out.cum) line_epilogue<256>(out, tcnt, o, u, L, x, threadIdx.x, sh);
        __syncthreads();
    }
}

// shared memory of one xl line sort
struct XlSmem {
    int hist[256];
    int base[256];
    int wcnt[8][256];
    int sh[8];
};

// LSD radix sort (8-bit digits over col_bits) + RLE of one very long segment
// seg[o, o + L) by a 256-thread CTA, ping-ponging with gkeys[2 o, ...);
// returns the run count (runs in tcol / tcnt at o)
template <typename K>
GSAP_DEV int xl_sort_line(K *__restrict__ seg, int o, int L, int col_bits, int *__restrict__ tcol,
                          int *__restrict__ tcnt, K *__restrict__ gkeys, int *__restrict__ ghp, XlSmem &S) {
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const unsigned lt = (1u << lane) - 1u;
    const int shift0 = sizeof(K) == 8 ? 32 : 0;
    K *src = seg + o;
    K *dst = gkeys + 2 * (size_t)o;
    for (int sbit = 0; sbit < col_bits; sbit += 8) {
        const int shift = shift0 + sbit;
        S.hist[tid] = 0;
        __syncthreads();
        for (int i = tid; i < L; i += 256) atomicAdd(&S.hist[(int)((src[i] >> shift) & 255)], 1);
        __syncthreads();
        {
            const int h = S.hist[tid];
            int x2 = h;
#pragma unroll
            for (int q = 1; q < 32; q <<= 1) {
                const int t = __shfl_up_sync(FULL, x2, q);
                if (lane >= q) x2 += t;
            }
            if (lane == 31) S.sh[w] = x2;
            __syncthreads();
            int wb = 0;
            for (int q = 0; q < 8; ++q)
                if (q < w) wb += S.sh[q];
            S.base[tid] = wb + x2 - h;
            __syncthreads();
        }
        for (int t0 = 0; t0 < L; t0 += 256) {
            const int i = t0 + tid;
            const bool valid = i < L;
            const K k = valid ? src[i] : (K)0;
            const int d = valid ? (int)((k >> shift) & 255) : 256;
#pragma unroll
            for (int q = 0; q < 8; ++q) S.wcnt[q][tid] = 0;
            __syncthreads();
            const unsigned peers = __match_any_sync(FULL, d);
            const int rank = __popc(peers & lt);
            if (valid && lane == __ffs(peers) - 1) S.wcnt[w][d] = __popc(peers);
            __syncthreads();
            // per digit (thread tid = digit): prefix over warps, then advance the base
            {
                int run = 0;
                for (int q = 0; q < 8; ++q) {
                    const int c = S.wcnt[q][tid];
                    S.wcnt[q][tid] = run;
                    run += c;
                }
                S.hist[tid] = run;   // this tile's count of digit tid
            }
            __syncthreads();
            if (valid) dst[S.base[d] + S.wcnt[w][d] + rank] = k;
            __syncthreads();
            S.base[tid] += S.hist[tid];
            __syncthreads();
        }
        K *t = src;
        src = dst;
        dst = t;
        __syncthreads();
    }
    return rle_runs<K, 256>(src, L, ghp + 2 * (size_t)o, tcol + o, tcnt + o, tid, S.sh);
}

// 4d. very long segments (> SegCta::CAP): one CTA each, LSD radix sort of the
// segment over the key's block bits in global memory (8-bit digits; a tile of
// 256 keys ranked stably with __match_any_sync per warp + per-warp digit
// counts), ping-pong between the segment and its scratch region, then RLE.
template <typename K>
__global__ void __launch_bounds__(256) k_segsort_xl(const int *__restrict__ off, K *__restrict__ seg,
                                                    const int *__restrict__ listC, const int *__restrict__ counters,
                                                    int col_bits, int *__restrict__ tcol, int *__restrict__ tcnt,
                                                    int *__restrict__ nnz, K *__restrict__ gkeys, int *__restrict__ ghp,
                                                    LineOut out) {
    __shared__ XlSmem S;
    const int n_lines = counters[1];
    for (int li = blockIdx.x; li < n_lines; li += gridDim.x) {
        const int x = listC[li];
        const int o = off[x], L = off[x + 1] - o;
        if (L <= SegCta<K>::CAP) continue;   // handled by k_segsort_cta
        const int u = xl_sort_line<K>(seg, o, L, col_bits, tcol, tcnt, gkeys, ghp, S);
        if (threadIdx.x == 0) nnz[x] = u;
        if (out.cum) line_epilogue<256>(out, tcnt, o, u, L, x, threadIdx.x, S.sh);
        __syncthreads();
    }
}

}  // namespace gsap
