// coop.cuh -- the sparse-regime blockmodel rebuild (Alg. 2, P:268-283 3.4) as
// ONE persistent kernel with grid-wide barriers, for graphs small enough that
// the multi-kernel path of segsort.cuh is bound by launch latency and per-
// kernel ramp/tail rather than by work (e.g. 20K vertices, 0.5M edges:
// ~20 launches of a few microseconds of work each).
//
// Same algorithm and the same bits as rebuild_sparse (both sides -- rows of
// M from the out-CSR, columns of M from the in-CSC -- in the same phases):
//   P0 zero line lengths / cursors / degrees          | barrier
//   P1 line lengths (counting sort pass 1), dout, din  | barrier
//   P2 CTA 0 / 1 scan the row / column lengths into segment offsets and list
//      the long lines; the other CTAs write rcp = 1 / (d + B)  | barrier
//   P3 scatter the neighbour blocks into their line's segment  | barrier
//   P4 per-line sort + run-length encoding: warps take the short lines,
//      CTAs the long ones (shared-memory radix <= CAP, global radix beyond);
//      the runs stay at the line's segment offset (padded CSR / CSC: the
//      same warp / CTA writes cum, end[x] and zero counts in the padding).
// The grid is sized to be co-resident (occupancy x SMs) and launched
// cooperatively; the barrier is the usual arrive-counter + generation flag.
#pragma once

#include "segsort.cuh"

namespace gsap {

struct CoopSide {
    const int *__restrict__ gptr;   // graph lines: out-CSR rowptr / in-CSC cscptr
    const int *__restrict__ gidx;   // the neighbours' blocks (neighbour-block cache nbo / nbi)
    const int *__restrict__ gw;     // weights or nullptr
    int *len, *cur, *nnz, *listC;   // [B + 1] line scratch
    int *off;                       // out: [B + 1] segment offsets = line pointers (padded)
    void *seg;                      // K[E] segment keys
    int *tcol, *tcnt;               // out: [E] runs (block, count) at the segment offsets
    void *xl_keys;                  // K[2E] global radix scratch
    int *xl_hp;                     // [2E]
    int *cum, *end, *deg;           // out: in-line prefix [E], line ends [B], line sums [B]
};

struct CoopArgs {
    int V, B, col_bits;
    const int *__restrict__ b;
    const int *__restrict__ kout;
    const int *__restrict__ kin;
    CoopSide sd[2];
    double *rcp;
    int *d_nnz;
    int *nlong;       // [3] long lines per side, short-line work counter
    unsigned *bar;    // [2] barrier: arrivals, generation
    // the neighbour-block cache update of the MOVE batch before this rebuild
    // (k_nb_update's work, done in P1 -- before the scatter reads the cache):
    // moved == nullptr: none pending
    const int *moved, *moved_cnt, *movedb, *rowptr, *cscptr, *csc2csr, *csr2csc;
    int *nbo, *nbi;
};

GSAP_DEV void grid_sync(unsigned *bar) {
    __syncthreads();
    if (threadIdx.x == 0) {
        volatile unsigned *gen = bar + 1;
        const unsigned g = *gen;
        __threadfence();
        if (atomicAdd(bar, 1u) == gridDim.x - 1) {
            atomicExch(bar, 0u);
            __threadfence();
            atomicAdd(bar + 1, 1u);
        } else {
            while (*gen == g) __nanosleep(32);
        }
        __threadfence();
    }
    __syncthreads();
}

// exclusive scan of in[0, n) into out[0, n], out[n] = total, by one 256-thread
// CTA; lines longer than SEG_WARP_MAX are appended to list (count in *nlist)
GSAP_DEV void cta_scan_lines(const int *in, int *out, int n, int *list, int *nlist, int *sh) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int carry = 0;
    for (int base = 0; base < n; base += 256 * 8) {
        int v[8], sm = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int idx = base + threadIdx.x * 8 + i;
            v[i] = idx < n ? in[idx] : 0;
            sm += v[i];
            if (list && v[i] > SEG_WARP_MAX) list[atomicAdd(nlist, 1)] = idx;
        }
        const int x = warp_incl_scan(sm);
        if (lane == 31) sh[w] = x;
        __syncthreads();
        int wb = 0, tot = 0;
        for (int i = 0; i < 8; ++i) {
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

// shared memory of the persistent rebuild: the union of its phases
template <typename K>
union CoopSmem {
    struct {
        K keys[SEG_WARPS][SEG_WARP_MAX];
        int hp[SEG_WARPS][SEG_WARP_MAX];
        unsigned cntp[SEG_WARPS][8 * 32];
    } warp;
    struct {
        K keys[2][SegCta<K>::CAP];
        unsigned cntp[8 * 256];
        unsigned wsum[8 * 8];
        int sh[8];
    } cta;
    XlSmem xl;
    int scan[8];
};

#ifdef GSAP_COOP_PROF   // experiment builds only (tools/build_variant.sh): per-phase times by printf
__device__ unsigned long long g_coop_t[8];
__device__ unsigned g_coop_done;
GSAP_DEV unsigned long long coop_now() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
#define COOP_MARK(i) \
    if (blockIdx.x == 0 && threadIdx.x == 0) g_coop_t[i] = coop_now();
#else
#define COOP_MARK(i)
#endif

template <typename K>
__global__ void __launch_bounds__(256) k_rebuild_coop(CoopArgs a) {
    extern __shared__ __align__(16) unsigned char coop_raw[];
    CoopSmem<K> &S = *reinterpret_cast<CoopSmem<K> *>(coop_raw);
    const int B = a.B, V = a.V;
    const int gtid = blockIdx.x * blockDim.x + threadIdx.x, gthreads = gridDim.x * blockDim.x;
    const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
    const int gwarp = gtid >> 5, gwarps = gthreads >> 5;
    COOP_MARK(0)
    // P0
    for (int x = gtid; x <= B; x += gthreads) {
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            a.sd[q].len[x] = 0;
            a.sd[q].cur[x] = 0;
            if (x < B) a.sd[q].deg[x] = 0;
        }
    }
    if (gtid < 3) a.nlong[gtid] = 0;   // [0, 1] long lines per side, [2] P4a work counter
    grid_sync(a.bar);
    COOP_MARK(1)
    // P1
    for (int v = gtid; v < V; v += gthreads) {
        const int x = __ldg(a.b + v);
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const int d = __ldg(a.sd[q].gptr + v + 1) - __ldg(a.sd[q].gptr + v);
            if (d) atomicAdd(a.sd[q].len + x, d);
        }
        const int ko = __ldg(a.kout + v), ki = __ldg(a.kin + v);
        if (ko) atomicAdd(a.sd[0].deg + x, ko);
        if (ki) atomicAdd(a.sd[1].deg + x, ki);
    }
    if (a.moved) {   // the pending cache update, one warp per moved vertex (as k_nb_update)
        const int n = *a.moved_cnt;
        for (int k = gwarp; k < n; k += gwarps) {
            const int v = a.moved[k], x = a.movedb[k];
            const int q1 = __ldg(a.cscptr + v + 1), p1 = __ldg(a.rowptr + v + 1);
            for (int q = __ldg(a.cscptr + v) + lane; q < q1; q += 32) a.nbo[__ldg(a.csc2csr + q)] = x;
            for (int p = __ldg(a.rowptr + v) + lane; p < p1; p += 32) a.nbi[__ldg(a.csr2csc + p)] = x;
        }
    }
    grid_sync(a.bar);
    COOP_MARK(2)
    // P2
    if (blockIdx.x < 2) {
        CoopSide &sd = a.sd[blockIdx.x];
        cta_scan_lines(sd.len, sd.off, B, sd.listC, a.nlong + blockIdx.x, S.scan);
    } else {
        for (int x = gtid - 2 * (int)blockDim.x; x < B; x += gthreads - 2 * (int)blockDim.x)
            a.rcp[x] = 1.0 / ((double)a.sd[0].deg[x] + (double)a.sd[1].deg[x] + (double)B);
    }
    grid_sync(a.bar);
    COOP_MARK(3)
    // P3: scatter, 32 (side, vertex) tasks per warp step (segsort.cuh scatter_batched)
    {
        const ScatterSide<K> s0{a.sd[0].gptr, a.sd[0].gidx, a.sd[0].gw, a.sd[0].off, a.sd[0].cur,
                                reinterpret_cast<K *>(a.sd[0].seg)};
        const ScatterSide<K> s1{a.sd[1].gptr, a.sd[1].gidx, a.sd[1].gw, a.sd[1].off, a.sd[1].cur,
                                reinterpret_cast<K *>(a.sd[1].seg)};
        scatter_batched<K>(s0, s1, 2, V, a.b, gwarp, gwarps);
    }
    grid_sync(a.bar);
    COOP_MARK(4)
    // P4b: long lines first, one CTA each (static: CTA i takes long lines i, i + grid, ...)
    {
        const int n0 = a.nlong[0], n1 = a.nlong[1];
        for (int li = blockIdx.x; li < n0 + n1; li += gridDim.x) {
            const int q = li >= n0;
            const CoopSide &sd = a.sd[q];
            const int x = sd.listC[q ? li - n0 : li];
            const int o = sd.off[x], L = sd.off[x + 1] - o;
            K *seg = reinterpret_cast<K *>(sd.seg);
            const LineOut out{sd.cum, sd.end, sd.deg};
            int u;
            if (L <= SegCta<K>::CAP) {
                K *keys = cta_sort(seg + o, L, S.cta.keys[0], S.cta.keys[1], a.col_bits, S.cta.cntp, S.cta.wsum);
                int *hp = reinterpret_cast<int *>(keys == S.cta.keys[0] ? S.cta.keys[1] : S.cta.keys[0]);
                u = rle_runs<K, 256>(keys, L, hp, sd.tcol + o, sd.tcnt + o, threadIdx.x, S.cta.sh);
                line_epilogue<256>(out, sd.tcnt, o, u, L, x, threadIdx.x, S.cta.sh);
            } else {
                u = xl_sort_line<K>(seg, o, L, a.col_bits, sd.tcol, sd.tcnt, reinterpret_cast<K *>(sd.xl_keys),
                                    sd.xl_hp, S.xl);
                line_epilogue<256>(out, sd.tcnt, o, u, L, x, threadIdx.x, S.xl.sh);
            }
            if (threadIdx.x == 0) sd.nnz[x] = u;
            __syncthreads();
        }
    }
    COOP_MARK(5)
    __syncthreads();   // the shared memory changes role
    // P4a: short lines, one warp each (bitonic + RLE in registers / shared
    // memory), fetched two at a time from a work counter: warps of CTAs that
    // sorted a long line first join late, the others keep going -- the phase
    // ends within ~one line of the slowest warp
    for (;;) {
        int t0 = 0;
        if (lane == 0) t0 = atomicAdd(a.nlong + 2, 2);
        t0 = __shfl_sync(FULL, t0, 0);
        if (t0 >= 2 * B) break;
        for (int task = t0; task < min(t0 + 2, 2 * B); ++task) {
            const int q = task >= B, x = q ? task - B : task;
            const CoopSide &sd = a.sd[q];
            const int o = sd.off[x], L = sd.off[x + 1] - o;
            if (L > SEG_WARP_MAX) continue;
            if (L == 0) {
                if (lane == 0) {
                    sd.nnz[x] = 0;
                    sd.end[x] = o;
                }
                continue;
            }
            const LineOut out{sd.cum, sd.end, sd.deg};
            const K *seg = reinterpret_cast<const K *>(sd.seg);
            if (L <= 128) {   // short lines: bitonic in registers, RLE in registers
                int u;
                if (L <= 32) u = warp_segsort_rle<K, 1>(seg + o, L, sd.tcol + o, sd.tcnt + o);
                else if (L <= 64) u = warp_segsort_rle<K, 2>(seg + o, L, sd.tcol + o, sd.tcnt + o);
                else u = warp_segsort_rle<K, 4>(seg + o, L, sd.tcol + o, sd.tcnt + o);
                if (lane == 0) sd.nnz[x] = u;
                line_epilogue<32>(out, sd.tcnt, o, u, L, x, lane, nullptr);
                continue;
            }
            int u;
            if (sizeof(K) == 4) {
                // 129..512 entries: one bucket pass + insertion sorts (segsort.cuh
                // warp_bucket_line), the padded output written directly
                u = warp_bucket_line<SEG_WARP_MAX>(reinterpret_cast<const unsigned *>(seg) + o, L, a.col_bits,
                                                   reinterpret_cast<unsigned *>(S.warp.keys[wl]), S.warp.hp[wl],
                                                   S.warp.cntp[wl], sd.tcol + o, sd.tcnt + o, sd.cum + o);
                if (lane == 0) {
                    sd.nnz[x] = u;
                    sd.end[x] = o + u;
                    sd.deg[x] = L;
                }
                continue;
            } else {
                int n = 1;
                while (n < L) n <<= 1;
                for (int i = lane; i < n; i += 32) S.warp.keys[wl][i] = i < L ? seg[o + i] : key_max<K>();
                __syncwarp();
                bitonic<K, 32>(S.warp.keys[wl], n, lane);
                u = rle_runs<K, 32>(S.warp.keys[wl], L, S.warp.hp[wl], sd.tcol + o, sd.tcnt + o, lane, nullptr);
            }
            if (lane == 0) sd.nnz[x] = u;
            line_epilogue<32>(out, sd.tcnt, o, u, L, x, lane, nullptr);
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *a.d_nnz = a.sd[0].off[B];   // the extent E (padding has cnt 0)
#ifdef GSAP_COOP_PROF
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        if (atomicAdd(&g_coop_done, 1u) == gridDim.x - 1) {
            const unsigned long long t6 = coop_now();
            g_coop_done = 0;
            printf("COOP B=%d nlong=%d,%d P0 %.2f P1 %.2f P2 %.2f P3 %.2f P4b0 %.2f P4 %.2f total %.2f us\n", B,
                   a.nlong[0], a.nlong[1], (g_coop_t[1] - g_coop_t[0]) * 1e-3, (g_coop_t[2] - g_coop_t[1]) * 1e-3,
                   (g_coop_t[3] - g_coop_t[2]) * 1e-3, (g_coop_t[4] - g_coop_t[3]) * 1e-3,
                   (g_coop_t[5] - g_coop_t[4]) * 1e-3, (t6 - g_coop_t[4]) * 1e-3, (t6 - g_coop_t[0]) * 1e-3);
        }
    }
#endif
}

}  // namespace gsap
