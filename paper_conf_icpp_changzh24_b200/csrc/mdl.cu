// mdl.cu -- the full description length, Eq. 1-2 (P:56-65 2.1; readings
// Z1-Z4, Z22):
//   S   = -sum_xy f(M_xy) + sum_x f(dout_x) + sum_y f(din_y),  f(m) = m ln m
//   MDL = E h(B^2/E) + V ln B + S,  h(x) = (1 + x) ln(1 + x) - x ln x.
// The data term is a fixed-chunk fp64 reduction (chunk = 2048 entries per
// CTA, then one ordered pass by the last CTA to finish), so it does not depend
// on the launch shape.  f(m) for m < FT_N comes from the double-double table
// (written in long double on the host), a log only beyond it.
#include <math.h>

#include <algorithm>

#include "internal.h"

namespace gsap {

constexpr int MDL_CHUNK = 2048;

GSAP_DEV double f_of(const double2 *__restrict__ ft, int m) {
    if (m <= 0) return 0.0;
    if (m < FT_N) {
        const double2 e = __ldg(ft + m);
        return e.x + e.y;
    }
    return fx((double)m);
}

__global__ void __launch_bounds__(256) k_mdl_partials(const int *__restrict__ cnt, const int *__restrict__ d_nnz,
                                                      const int *__restrict__ dout, const int *__restrict__ din,
                                                      int B, const double2 *__restrict__ ft,
                                                      double *__restrict__ partials, unsigned *__restrict__ arrivals,
                                                      double *__restrict__ out, DsumSpec ds, double *__restrict__ dsum) {
    __shared__ double sh[8];
    __shared__ bool last;
    const int nnz = *d_nnz;
    const long long base = (long long)blockIdx.x * MDL_CHUNK;
    double acc = 0.0;
    for (int k = threadIdx.x; k < MDL_CHUNK; k += 256) {
        const long long i = base + k;
        if (i < nnz) acc -= f_of(ft, cnt[i]);
        if (i < B) acc += f_of(ft, dout[i]) + f_of(ft, din[i]);
    }
    acc = warp_sum(acc);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < 8; ++w) t += sh[w];
        partials[blockIdx.x] = t;
        __threadfence();
        last = atomicAdd(arrivals, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    // the last CTA: one ordered pass over the partials (256 strided lanes, warp trees, 8 warp sums)
    double v = 0.0;
    for (int i = threadIdx.x; i < (int)gridDim.x; i += 256) v += *((volatile double *)(partials + i));
    v = warp_sum(v);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < 8; ++w) t += sh[w];
        *out = t;
        *arrivals = 0u;
    }
    if (ds.nbat == 0) return;
    // the iteration's dS sum: per batch the ordered pass of k_apply_sum over
    // its chunk partials (256 strided lanes, warp trees, 8 warp sums), added to
    // the running sum batch after batch -- the same operations in the same order
    double run = 0.0;
    if (ds.nch_first <= 32 && ds.nch_last <= 32 && ds.nbat <= 8) {
        // <= 32 partials per batch: only warp 0's tree is non-zero (the other
        // seven warp sums are +0.0), so warp k computes batch k's tree at once
        const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
        __syncthreads();
        if (w < ds.nbat) {
            const int n = w + 1 < ds.nbat ? ds.nch_first : ds.nch_last;
            double v2 = 0.0;
            if (lane < n) v2 += ds.part[(size_t)w * ds.stride + lane];
            v2 = warp_sum(v2);
            if (lane == 0) sh[w] = v2;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int k = 0; k < ds.nbat; ++k) {
                double t = 0.0;
                t += sh[k];
                for (int q = 1; q < 8; ++q) t += 0.0;
                run += t;
            }
            *dsum = run;
        }
        return;
    }
    for (int k = 0; k < ds.nbat; ++k) {
        const int n = k + 1 < ds.nbat ? ds.nch_first : ds.nch_last;
        double v2 = 0.0;
        for (int i = threadIdx.x; i < n; i += 256) v2 += ds.part[(size_t)k * ds.stride + i];
        v2 = warp_sum(v2);
        __syncthreads();
        if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = v2;
        __syncthreads();
        if (threadIdx.x == 0) {
            double t = 0.0;
            for (int w = 0; w < 8; ++w) t += sh[w];
            run += t;
        }
    }
    if (threadIdx.x == 0) *dsum = run;
}

// launches the reduction into c.scal[1] (no synchronisation)
void launch_data_term(Ctx &c, const DsumSpec *dsum) {
    cudaEvent_t ev = nullptr;
    kc_begin(c, c.k_mdl, &ev);
    // the extent of the cnt array: nnz <= E, or B^2 for the padded dense lines
    long long n = std::max<long long>(std::max<long long>(c.E, c.B), 1);
    if (c.dense_padded) n = std::max(n, (long long)c.B * c.B);
    const int nb = (int)((n + MDL_CHUNK - 1) / MDL_CHUNK);
    const DsumSpec none{nullptr, 0, 0, 0, 0};
    k_mdl_partials<<<nb, 256, 0, c.stream>>>(c.bm_cnt, c.d_nnz, c.dout, c.din, c.B, c.ft, c.partials,
                                             reinterpret_cast<unsigned *>(c.scal_i + 5), c.scal + 1,
                                             dsum ? *dsum : none, c.scal);
    c.launches += 1;
    GSAP_CHECK_LAUNCH();
    kc_end(c, c.k_mdl, ev, 0.0);
}

double device_data_term(Ctx &c) {
    launch_data_term(c);
    GSAP_CUDA(cudaMemcpyAsync(c.h_scal + 1, c.scal + 1, sizeof(double), cudaMemcpyDeviceToHost, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    return c.h_scal[1];
}

double model_term(long long W, int V, int B, int variant) {
    const double lnB = log((double)B);
    if (W <= 0) return (double)V * lnB;
    const double E = (double)W, x = (double)B * (double)B / E;
    const double t = variant == 1 ? E * (1.0 + x) * log1p(x) - x * log(x)
                                  : E * ((1.0 + x) * log1p(x) - x * log(x));
    return t + (double)V * lnB;
}

}  // namespace gsap
