// prims.cuh -- hand-written device-wide primitives for the blockmodel rebuild
// (Alg. 2, P:268-283 3.4: sort_by_key / segsort / prefix_scan / segreduce):
// a reduce-then-scan prefix sum and a stable LSD radix sort (8-bit digits,
// warp-level multisplit with __match_any_sync, tile-local reorder in shared
// memory so the global scatter is coalesced per digit run).
//
// Counts may live on the device (d_n != nullptr): grids are sized for n_max
// and every kernel reads the true n, so no host synchronisation is needed.
#pragma once

#include "common.cuh"

namespace gsap {

constexpr int PT_THREADS = 256;
constexpr int PT_ITEMS = 16;
constexpr int PT_TILE = PT_THREADS * PT_ITEMS;   // 4096
constexpr int RS_RADIX = 256;

GSAP_DEV int read_n(const int *d_n, int n_static) { return d_n ? *d_n : n_static; }

// exclusive block scan over PT_THREADS values (returns the block total too)
template <typename T>
GSAP_DEV T block_excl_scan(T v, T *total, T *sh /* >= 8 */) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    T x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const T t = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += t;
    }
    if (lane == 31) sh[w] = x;
    __syncthreads();
    T wbase = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < PT_THREADS / 32; ++i) {
        const T s = sh[i];
        if (i < w) wbase += s;
        tot += s;
    }
    __syncthreads();
    *total = tot;
    return wbase + x - v;
}

template <typename T>
__global__ void __launch_bounds__(PT_THREADS) k_tile_sums(const T *__restrict__ in, const int *d_n,
                                                          int n_static, T *__restrict__ sums) {
    __shared__ T sh[8];
    const int n = read_n(d_n, n_static);
    const long long base = (long long)blockIdx.x * PT_TILE;
    T acc = 0;
    for (int i = threadIdx.x; i < PT_TILE; i += PT_THREADS) {
        const long long idx = base + i;
        if (idx < n) acc += in[idx];
    }
    T tot;
    block_excl_scan<T>(acc, &tot, sh);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

// single CTA, in-place exclusive scan of a[0, m); *total = sum (nullable)
template <typename T>
__global__ void __launch_bounds__(PT_THREADS) k_scan_small(T *a, int m, T *total) {
    __shared__ T sh[8];
    T carry = 0;
    for (int base = 0; base < m; base += PT_THREADS * 4) {
        T v[4], s = 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int idx = base + threadIdx.x * 4 + i;
            v[i] = idx < m ? a[idx] : T(0);
            s += v[i];
        }
        T tot;
        T ex = block_excl_scan<T>(s, &tot, sh) + carry;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int idx = base + threadIdx.x * 4 + i;
            if (idx < m) a[idx] = ex;
            ex += v[i];
        }
        carry += tot;
    }
    if (total && threadIdx.x == 0) *total = carry;
}

// per tile: scan with the tile's offset (exclusive offsets from k_scan_small)
template <typename T, bool INCLUSIVE>
__global__ void __launch_bounds__(PT_THREADS) k_scan_tiles(const T *in, T *out,
                                                           const int *d_n, int n_static,
                                                           const T *offs) {
    __shared__ T buf[PT_TILE];
    __shared__ T sh[8];
    const int n = read_n(d_n, n_static);
    const long long base = (long long)blockIdx.x * PT_TILE;
    if (base >= n) return;
    for (int i = threadIdx.x; i < PT_TILE; i += PT_THREADS) {
        const long long idx = base + i;
        buf[i] = idx < n ? in[idx] : T(0);
    }
    __syncthreads();
    T v[PT_ITEMS], s = 0;
#pragma unroll
    for (int i = 0; i < PT_ITEMS; ++i) {
        v[i] = buf[threadIdx.x * PT_ITEMS + i];
        s += v[i];
    }
    T tot;
    T ex = block_excl_scan<T>(s, &tot, sh) + offs[blockIdx.x];
#pragma unroll
    for (int i = 0; i < PT_ITEMS; ++i) {
        if (INCLUSIVE) {
            ex += v[i];
            buf[threadIdx.x * PT_ITEMS + i] = ex;
        } else {
            buf[threadIdx.x * PT_ITEMS + i] = ex;
            ex += v[i];
        }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < PT_TILE; i += PT_THREADS) {
        const long long idx = base + i;
        if (idx < n) out[idx] = buf[i];
    }
}

// --------------------------------------------------------------- radix --
template <typename K>
GSAP_DEV int digit_of(K k, int shift) { return (int)((k >> shift) & (K)(RS_RADIX - 1)); }

template <typename K>
__global__ void __launch_bounds__(PT_THREADS) k_rs_upsweep(const K *__restrict__ keys, const int *d_n,
                                                           int n_static, int shift,
                                                           int *__restrict__ counts, int ntiles) {
    __shared__ int hist[RS_RADIX];
    const int n = read_n(d_n, n_static);
    hist[threadIdx.x] = 0;
    __syncthreads();
    const long long base = (long long)blockIdx.x * PT_TILE;
    for (int i = threadIdx.x; i < PT_TILE; i += PT_THREADS) {
        const long long idx = base + i;
        const int d = idx < n ? digit_of<K>(keys[idx], shift) : RS_RADIX;
        const unsigned peers = __match_any_sync(FULL, d);
        if (d < RS_RADIX && (int)(threadIdx.x & 31) == __ffs(peers) - 1)
            atomicAdd(&hist[d], __popc(peers));
    }
    __syncthreads();
    counts[(size_t)threadIdx.x * ntiles + blockIdx.x] = hist[threadIdx.x];
}

template <typename K, typename V, bool HAS_V>
__global__ void __launch_bounds__(PT_THREADS) k_rs_downsweep(const K *__restrict__ kin, K *__restrict__ kout,
                                                             const V *__restrict__ vin, V *__restrict__ vout,
                                                             const int *d_n, int n_static, int shift,
                                                             const int *__restrict__ offsets, int ntiles) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    K *skeys = reinterpret_cast<K *>(smem_raw);
    V *svals = reinterpret_cast<V *>(smem_raw + sizeof(K) * PT_TILE);
    __shared__ int whist[PT_THREADS / 32][RS_RADIX];
    __shared__ int tile_start[RS_RADIX];
    __shared__ int digit_base[RS_RADIX];
    __shared__ int sh[8];
    const int n = read_n(d_n, n_static);
    const long long base = (long long)blockIdx.x * PT_TILE;
    if (base >= n) return;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int i = 0; i < PT_THREADS / 32; ++i) whist[i][threadIdx.x] = 0;
    __syncthreads();
    K k[PT_ITEMS];
    int d[PT_ITEMS], loc[PT_ITEMS];
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int r = 0; r < PT_ITEMS; ++r) {
        const long long idx = base + w * (32 * PT_ITEMS) + r * 32 + lane;
        k[r] = idx < n ? kin[idx] : K(0);
        d[r] = idx < n ? digit_of<K>(k[r], shift) : RS_RADIX;
    }
#pragma unroll
    for (int r = 0; r < PT_ITEMS; ++r) {
        const unsigned peers = __match_any_sync(FULL, d[r]);
        const int cur = d[r] < RS_RADIX ? whist[w][d[r]] : 0;
        loc[r] = cur + __popc(peers & lt);
        __syncwarp();
        if (d[r] < RS_RADIX && lane == __ffs(peers) - 1) whist[w][d[r]] = cur + __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    {
        const int t = threadIdx.x;   // digit
        int run = 0;
#pragma unroll
        for (int i = 0; i < PT_THREADS / 32; ++i) {
            const int c = whist[i][t];
            whist[i][t] = run;
            run += c;
        }
        int tot;
        tile_start[t] = block_excl_scan<int>(run, &tot, sh);
        digit_base[t] = offsets[(size_t)t * ntiles + blockIdx.x];
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < PT_ITEMS; ++r) {
        if (d[r] < RS_RADIX) {
            const int p = tile_start[d[r]] + whist[w][d[r]] + loc[r];
            skeys[p] = k[r];
            if (HAS_V) svals[p] = vin[base + w * (32 * PT_ITEMS) + r * 32 + lane];
        }
    }
    __syncthreads();
    const int cnt = (int)min((long long)PT_TILE, (long long)n - base);
    for (int i = threadIdx.x; i < cnt; i += PT_THREADS) {
        const K key = skeys[i];
        const int dd = digit_of<K>(key, shift);
        const long long g = (long long)digit_base[dd] + (i - tile_start[dd]);
        kout[g] = key;
        if (HAS_V) vout[g] = svals[i];
    }
}

// one CTA scans everything (small arrays: one launch instead of three)
constexpr int SS_THREADS = 1024, SS_ITEMS = 8;
template <typename T, bool INCLUSIVE>
__global__ void __launch_bounds__(SS_THREADS) k_scan_single(const T *in, T *out, const int *d_n, int n_static,
                                                             T *total) {
    __shared__ T sh[SS_THREADS / 32];
    const int n = read_n(d_n, n_static);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    T carry = 0;
    for (int base = 0; base < n; base += SS_THREADS * SS_ITEMS) {
        T v[SS_ITEMS], s = 0;
#pragma unroll
        for (int i = 0; i < SS_ITEMS; ++i) {
            const int idx = base + threadIdx.x * SS_ITEMS + i;
            v[i] = idx < n ? in[idx] : T(0);
            s += v[i];
        }
        T x = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const T t = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += t;
        }
        if (lane == 31) sh[w] = x;
        __syncthreads();
        T wb = 0, tot = 0;
        for (int i = 0; i < SS_THREADS / 32; ++i) {
            const T q = sh[i];
            if (i < w) wb += q;
            tot += q;
        }
        __syncthreads();
        T ex = carry + wb + x - s;
#pragma unroll
        for (int i = 0; i < SS_ITEMS; ++i) {
            const int idx = base + threadIdx.x * SS_ITEMS + i;
            if (INCLUSIVE) ex += v[i];
            if (idx < n) out[idx] = ex;
            if (!INCLUSIVE) ex += v[i];
        }
        carry += tot;
    }
    if (total && threadIdx.x == 0) *total = carry;
}

// host side -----------------------------------------------------------------
struct Launcher {
    cudaStream_t stream;
    long long *launches;   // incremented per kernel launch
};

inline int tiles_for(long long n) { return (int)((n + PT_TILE - 1) / PT_TILE); }

// exclusive / inclusive scan of in[0, n) into out; tmp >= tiles_for(n_max) + 1 elements
template <typename T>
void device_scan(const T *in, T *out, const int *d_n, int n_max, bool inclusive, T *tmp,
                 T *total, const Launcher &L) {
    const int nt = tiles_for(n_max);
    if (nt == 0) return;
    if (n_max <= 4 * SS_THREADS * SS_ITEMS) {
        if (inclusive) k_scan_single<T, true><<<1, SS_THREADS, 0, L.stream>>>(in, out, d_n, n_max, total);
        else k_scan_single<T, false><<<1, SS_THREADS, 0, L.stream>>>(in, out, d_n, n_max, total);
        *L.launches += 1;
        return;
    }
    k_tile_sums<T><<<nt, PT_THREADS, 0, L.stream>>>(in, d_n, n_max, tmp);
    k_scan_small<T><<<1, PT_THREADS, 0, L.stream>>>(tmp, nt, total);
    if (inclusive)
        k_scan_tiles<T, true><<<nt, PT_THREADS, 0, L.stream>>>(in, out, d_n, n_max, tmp);
    else
        k_scan_tiles<T, false><<<nt, PT_THREADS, 0, L.stream>>>(in, out, d_n, n_max, tmp);
    *L.launches += 3;
}

// stable LSD radix sort of (keys, vals) on bits [0, bits); buffers ping-pong;
// returns 1 if the result is in (k1, v1), 0 if in (k0, v0).
// counts: RS_RADIX * tiles_for(n_max) ints; scan_tmp: tiles_for(RS_RADIX*tiles)+1 ints.
template <typename K, typename V, bool HAS_V>
int radix_sort(K *k0, K *k1, V *v0, V *v1, const int *d_n, int n_max, int bits, int *counts,
               int *scan_tmp, const Launcher &L) {
    const int nt = tiles_for(n_max);
    if (nt == 0 || bits <= 0) return 0;
    const size_t smem = sizeof(K) * PT_TILE + (HAS_V ? sizeof(V) * PT_TILE : 0);
    per_device((const void *)k_rs_downsweep<K, V, HAS_V>, [&] {
        GSAP_CUDA(cudaFuncSetAttribute(k_rs_downsweep<K, V, HAS_V>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem));
        return 1;
    });
    int cur = 0;
    for (int shift = 0; shift < bits; shift += 8) {
        K *ks = cur ? k1 : k0;
        K *kd = cur ? k0 : k1;
        V *vs = cur ? v1 : v0;
        V *vd = cur ? v0 : v1;
        k_rs_upsweep<K><<<nt, PT_THREADS, 0, L.stream>>>(ks, d_n, n_max, shift, counts, nt);
        ++*L.launches;
        device_scan<int>(counts, counts, nullptr, RS_RADIX * nt, false, scan_tmp, nullptr, L);
        k_rs_downsweep<K, V, HAS_V><<<nt, PT_THREADS, smem, L.stream>>>(ks, kd, vs, vd, d_n, n_max, shift,
                                                                        counts, nt);
        ++*L.launches;
        cur ^= 1;
    }
    return cur;
}

}  // namespace gsap
