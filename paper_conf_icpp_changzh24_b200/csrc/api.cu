// api.cu -- the C-ABI (include/gsap.h): context management, argument
// marshalling, and the thin host driver of SBP (P:137-141 3 Fig. 2): merge ->
// batched MCMC (Table 2) -> golden-section search over B (P:34 1,
// P:328 4.3; readings Z19-Z21), which stays on the host as in the paper.
#include <math.h>
#include <string.h>

#include <algorithm>
#include <cstdlib>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <mutex>
#include <new>
#include <vector>

#include "internal.h"

struct gsap_ctx {
    gsap::Ctx c;
};

using namespace gsap;

static thread_local std::string g_err;

#define API_TRY try {
#define API_CATCH                                      \
    }                                                  \
    catch (const Error &e) {                           \
        g_err = e.msg;                                 \
        return e.code;                                 \
    }                                                  \
    catch (const std::bad_alloc &) {                   \
        g_err = "host allocation failed";              \
        return GSAP_ENOMEM;                            \
    }                                                  \
    catch (const std::exception &e) {                  \
        g_err = e.what();                              \
        return GSAP_EINVAL;                            \
    }                                                  \
    catch (...) {                                      \
        g_err = "unknown error";                       \
        return GSAP_EINVAL;                            \
    }                                                  \
    return GSAP_OK;

#define REQUIRE(cond, code, msg)          \
    do {                                  \
        if (!(cond)) throw Error{code, msg}; \
    } while (0)

namespace gsap {

// ------------------------------------------------------- event timing --
static cudaEvent_t ev_get(KClass &k) {
    if (!k.pool.empty()) {
        cudaEvent_t e = k.pool.back();
        k.pool.pop_back();
        return e;
    }
    cudaEvent_t e;
    GSAP_CUDA(cudaEventCreate(&e));
    return e;
}

static void ev_record(Ctx &c, cudaEvent_t e) {
    if (c.capturing) GSAP_CUDA(cudaEventRecordWithFlags(e, c.stream, cudaEventRecordExternal));
    else GSAP_CUDA(cudaEventRecord(e, c.stream));
}

void kc_begin(Ctx &c, KClass &k, cudaEvent_t *ev) {
    *ev = nullptr;
    if (!c.prm.profile) return;
    *ev = ev_get(k);
    ev_record(c, *ev);
}

void kc_end(Ctx &c, KClass &k, cudaEvent_t ev, double bytes) {
    if (c.capturing) {   // accounted per graph launch (graph_account)
        if (ev) {
            cudaEvent_t e2 = ev_get(k);
            ev_record(c, e2);
            c.graph_ev.push_back(GraphEv{&k, ev, e2, bytes});
        } else {
            c.graph_ev.push_back(GraphEv{&k, nullptr, nullptr, bytes});
        }
        return;
    }
    k.launches += 1;
    k.bytes += bytes;
    if (!ev) return;
    cudaEvent_t e2 = ev_get(k);
    ev_record(c, e2);
    k.pending.emplace_back(ev, e2);
    if (k.pending.size() > 4096) kc_resolve(c, k);
}

// after one (synchronised) launch of a captured graph: account its kernel classes
static void graph_account(Ctx &c) {
    for (auto &g : c.graph_ev) {
        g.k->launches += 1;
        g.k->bytes += g.bytes;
        if (g.e0) {
            float ms = 0.f;
            GSAP_CUDA(cudaEventElapsedTime(&ms, g.e0, g.e1));
            g.k->ms += ms;
        }
    }
}

static void graph_release_events(Ctx &c) {
    for (auto &g : c.graph_ev) {
        if (g.e0) {
            g.k->pool.push_back(g.e0);
            g.k->pool.push_back(g.e1);
        }
    }
    c.graph_ev.clear();
}

// profile mode outside graph capture: one launch of a role timed on `st`
// (the MOVE roles run concurrently, so each is measured on its own stream)
cudaEvent_t role_begin(Ctx &c, KClass &k, cudaStream_t st) {
    if (!c.prm.profile || c.capturing) return nullptr;
    cudaEvent_t e = ev_get(k);
    GSAP_CUDA(cudaEventRecord(e, st));
    return e;
}

void role_end(Ctx &c, KClass &k, cudaEvent_t e0, cudaStream_t st) {
    if (!e0) return;
    cudaEvent_t e1 = ev_get(k);
    GSAP_CUDA(cudaEventRecord(e1, st));
    k.launches += 1;
    k.pending.emplace_back(e0, e1);
    if (k.pending.size() > 4096) kc_resolve(c, k);
}

void kc_resolve(Ctx &c, KClass &k) {
    (void)c;
    for (auto &p : k.pending) {
        GSAP_CUDA(cudaEventSynchronize(p.second));
        float ms = 0.f;
        GSAP_CUDA(cudaEventElapsedTime(&ms, p.first, p.second));
        k.ms += ms;
        k.pool.push_back(p.first);
        k.pool.push_back(p.second);
    }
    k.pending.clear();
}

}  // namespace gsap

int gsap::per_device(const void *key, const std::function<int()> &f) {
    int dev = 0;
    GSAP_CUDA(cudaGetDevice(&dev));
    static std::mutex mu;
    static std::map<std::pair<const void *, int>, int> cache;
    std::lock_guard<std::mutex> g(mu);
    const auto it = cache.find({key, dev});
    if (it != cache.end()) return it->second;
    const int v = f();
    cache[{key, dev}] = v;
    return v;
}

static bool is_dev(const void *p) {
    if (!p) return false;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// dst: host or device; src: device.  Complete on return (a device output is
// then safe on any stream of the caller: no ordering against c.stream needed)
static void copy_out(Ctx &c, void *dst, const void *src, size_t bytes) {
    if (!dst || !bytes) return;
    GSAP_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDefault, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
}

// src: host or device -> a device pointer (src itself, or staged into `scratch`)
template <typename T>
static const T *stage_in(Ctx &c, const T *src, size_t n, T *scratch) {
    if (!src || is_dev(src)) return src;
    if (n) GSAP_CUDA(cudaMemcpyAsync(scratch, src, n * sizeof(T), cudaMemcpyHostToDevice, c.stream));
    return scratch;
}

template <typename T>
static std::vector<T> to_host(const T *src, size_t n) {
    std::vector<T> h(n);
    if (n) GSAP_CUDA(cudaMemcpy(h.data(), src, n * sizeof(T), cudaMemcpyDefault));
    return h;
}

// one attribute query per device (cudaGetDeviceProperties fills the whole
// struct and was seen taking tens of ms inside gsap_partition's create)
static void check_sm100() {
    const int major = per_device((const void *)&check_sm100, [] {
        int dev = 0, mj = 0;
        GSAP_CUDA(cudaGetDevice(&dev));
        GSAP_CUDA(cudaDeviceGetAttribute(&mj, cudaDevAttrComputeCapabilityMajor, dev));
        return mj;
    });
    REQUIRE(major == 10, GSAP_EUNSUPPORTED, "libgsap is built for sm_100a (B200) only");
}

// The arena of the last destroyed context is kept (one per process) and
// handed to the next context of the same device that fits in it: repeated
// gsap_partition calls skip cudaMalloc / cudaFree of hundreds of MB
// (measured 3-14 ms and 4-6 ms per call at 20K-HH).  No buffer relies on
// fresh memory contents (everything is initialised explicitly).
namespace {
std::mutex g_arena_mu;
struct {
    void *p = nullptr;
    size_t bytes = 0;
    int dev = -1;
} g_arena_cache;
}  // namespace

static void *arena_take(int dev, size_t need, size_t *got) {
    {
        std::lock_guard<std::mutex> g(g_arena_mu);
        if (g_arena_cache.p && g_arena_cache.dev == dev && g_arena_cache.bytes >= need &&
            g_arena_cache.bytes <= 2 * need + (64u << 20)) {
            void *p = g_arena_cache.p;
            *got = g_arena_cache.bytes;
            g_arena_cache.p = nullptr;
            return p;
        }
    }
    return nullptr;
}

static void arena_give(void *p, size_t bytes, int dev) {
    void *drop = nullptr;
    {
        std::lock_guard<std::mutex> g(g_arena_mu);
        // keep the newest: the next create is most likely the same workload (keeping
        // the larger one made every later create of a smaller graph pay a
        // cudaMalloc + cudaFree -- e.g. the bench's 20K e2e calls after its 2M states)
        drop = g_arena_cache.p;
        g_arena_cache.p = p;
        g_arena_cache.bytes = bytes;
        g_arena_cache.dev = dev;
    }
    if (drop) cudaFree(drop);
}

static void drop_mcmc_exec(Ctx &c) {
    if (c.mcmc_exec) cudaGraphExecDestroy(c.mcmc_exec);
    c.mcmc_exec = nullptr;
    c.mcmc_exec_mode = 0;
}

// the executable graph of an MCMC phase: the cached one of the previous phase
// updated in place when the topology matches (kernel parameters, grid sizes,
// the regime's B all change between rounds; the node structure only with the
// regime), else a fresh instantiation
static cudaGraphExec_t mcmc_exec_for(Ctx &c, cudaGraph_t graph, int mode) {
    static const bool no_update = getenv("GSAP_NO_EXEC_UPDATE") != nullptr;   // A/B switch
    if (c.mcmc_exec && c.mcmc_exec_mode == mode && !no_update) {
        cudaGraphExecUpdateResultInfo info;
        if (cudaGraphExecUpdate(c.mcmc_exec, graph, &info) == cudaSuccess) return c.mcmc_exec;
        cudaGetLastError();   // clear the update's error state
    }
    drop_mcmc_exec(c);
    GSAP_CUDA(cudaGraphInstantiate(&c.mcmc_exec, graph, 0));
    c.mcmc_exec_mode = mode;
    return c.mcmc_exec;
}

static void free_ctx(Ctx &c) {
    drop_mcmc_exec(c);
    if (c.arena) {
        if (c.stream) cudaStreamSynchronize(c.stream);
        if (c.side) cudaStreamSynchronize(c.side);
        arena_give(c.arena, c.arena_bytes, c.dev);
    }
    c.arena = nullptr;
    if (c.h_scal) cudaFreeHost(c.h_scal);
    if (c.h_int) cudaFreeHost(c.h_int);
    for (KClass *k : {&c.k_move, &c.k_rebuild, &c.k_merge, &c.k_mdl, &c.k_comm, &c.k_groups, &c.k_warps}) {
        for (auto &p : k->pending) {
            cudaEventDestroy(p.first);
            cudaEventDestroy(p.second);
        }
        for (auto e : k->pool) cudaEventDestroy(e);
    }
    try {
        comm_destroy(c);
    } catch (...) {
    }
    if (c.own_stream && c.stream) cudaStreamDestroy(c.stream);
    if (c.side) cudaStreamDestroy(c.side);
    if (c.ev_fork) cudaEventDestroy(c.ev_fork);
    if (c.ev_join) cudaEventDestroy(c.ev_join);
    if (c.ev_nb) cudaEventDestroy(c.ev_nb);
    if (c.ev_apply) cudaEventDestroy(c.ev_apply);
    if (c.ev_rb_fork) cudaEventDestroy(c.ev_rb_fork);
    if (c.ev_rb_join) cudaEventDestroy(c.ev_rb_join);
}

// one device allocation per context, carved into aligned sub-buffers
struct Arena {
    char *base = nullptr;   // nullptr: measuring pass
    size_t off = 0;
    template <typename T>
    T *take(size_t n) {
        off = (off + 255) & ~(size_t)255;
        T *p = base ? reinterpret_cast<T *>(base + off) : nullptr;
        off += std::max<size_t>(n, 1) * sizeof(T);
        return p;
    }
};

static int log2_ceil_h(long long x) {
    int l = 0;
    while ((1LL << l) < x) ++l;
    return l;
}

// ----------------------------------------------------------- create ----
static void create_impl(Ctx &c, int32_t V, const int64_t *rowptr, const int32_t *col, const int32_t *wgt,
                        const gsap_params *params, const gsap_dist *dist, void *stream) {
    REQUIRE(V >= 1, GSAP_EINVAL, "V must be >= 1");
    REQUIRE(rowptr && (col || true), GSAP_EINVAL, "rowptr is NULL");
    const bool tm = getenv("GSAP_TIMING") != nullptr;
    auto t_prev = std::chrono::steady_clock::now();
    auto mark = [&](const char *what) {
        if (!tm) return;
        cudaDeviceSynchronize();
        const auto t = std::chrono::steady_clock::now();
        fprintf(stderr, "[gsap] create %-12s %.3f ms\n", what, std::chrono::duration<double, std::milli>(t - t_prev).count());
        t_prev = t;
    };
    check_sm100();
    if (params) c.prm = *params;
    else gsap_default_params(&c.prm);
    REQUIRE(c.prm.num_batches >= 1 && c.prm.max_nodal_itr >= 1 && c.prm.window >= 1, GSAP_EINVAL,
            "num_batches, max_nodal_itr and window must be >= 1");
    REQUIRE(c.prm.num_proposals >= 1 && c.prm.num_proposals <= 32, GSAP_EINVAL, "num_proposals in [1, 32]");
    // stage + validate the CSR on the host
    std::vector<int64_t> rp = to_host(rowptr, (size_t)V + 1);
    REQUIRE(rp[0] == 0, GSAP_EINVAL, "rowptr[0] must be 0");
    for (int v = 0; v < V; ++v) REQUIRE(rp[v + 1] >= rp[v], GSAP_EINVAL, "rowptr must be non-decreasing");
    const int64_t E64 = rp[V];
    REQUIRE(E64 < (1LL << 30), GSAP_EUNSUPPORTED, "more than 2^30 edges");
    REQUIRE(E64 == 0 || col, GSAP_EINVAL, "col is NULL");
    const int E = (int)E64;
    std::vector<int32_t> hc = to_host(col, (size_t)E);
    std::vector<int32_t> hw;
    long long W = 0;
    for (int e = 0; e < E; ++e) REQUIRE(hc[e] >= 0 && hc[e] < V, GSAP_EINVAL, "col out of range");
    if (wgt) {
        hw = to_host(wgt, (size_t)E);
        for (int e = 0; e < E; ++e) {
            REQUIRE(hw[e] >= 1, GSAP_EINVAL, "weights must be >= 1");
            W += hw[e];
        }
    } else {
        W = E;
    }
    REQUIRE(W < (1LL << 30), GSAP_EUNSUPPORTED, "total edge weight must be < 2^30");
    c.V = V;
    c.E = E;
    c.W = W;
    c.weighted = wgt != nullptr;
    mark("validate");
    if (stream) {
        c.stream = (cudaStream_t)stream;
    } else {
        GSAP_CUDA(cudaStreamCreateWithFlags(&c.stream, cudaStreamNonBlocking));
        c.own_stream = true;
    }
    GSAP_CUDA(cudaStreamCreateWithFlags(&c.side, cudaStreamNonBlocking));
    GSAP_CUDA(cudaEventCreateWithFlags(&c.ev_fork, cudaEventDisableTiming));
    GSAP_CUDA(cudaEventCreateWithFlags(&c.ev_join, cudaEventDisableTiming));
    GSAP_CUDA(cudaEventCreateWithFlags(&c.ev_nb, cudaEventDisableTiming));
    GSAP_CUDA(cudaEventCreateWithFlags(&c.ev_apply, cudaEventDisableTiming));
    GSAP_CUDA(cudaEventCreateWithFlags(&c.ev_rb_fork, cudaEventDisableTiming));
    GSAP_CUDA(cudaEventCreateWithFlags(&c.ev_rb_join, cudaEventDisableTiming));
    GSAP_CUDA(cudaGetDevice(&c.dev));
    comm_init(c, dist);
    if (const char *tg = getenv("GSAP_TEST_GRID")) c.test_grid = std::max(0, atoi(tg));
    REQUIRE(c.prm.sim_ranks >= 0 && c.prm.sim_ranks <= 64, GSAP_EINVAL, "sim_ranks in [0, 64]");
    REQUIRE(c.prm.proposal_mode == 0 || c.prm.proposal_mode == 1, GSAP_EINVAL, "proposal_mode is 0 or 1");
    REQUIRE(c.prm.line_sort == 0 || c.prm.line_sort == 1, GSAP_EINVAL, "line_sort is 0 or 1");
    if (c.nranks > 1 || c.prm.sim_ranks > 1) c.prm.cuda_graphs = 0;   // the sliced batch path (move_batch)
    mark("streams");
    // host-side static info
    c.h_rowptr.resize((size_t)V + 1);
    for (int v = 0; v <= V; ++v) c.h_rowptr[v] = (int)rp[v];
    c.h_cscptr.assign((size_t)V + 1, 0);
    for (int e = 0; e < E; ++e) c.h_cscptr[hc[e] + 1]++;
    for (int v = 0; v < V; ++v) c.h_cscptr[v + 1] += c.h_cscptr[v];
    int kmax_big = 0;
    for (int v = 0; v < V; ++v) {
        const int k = (c.h_rowptr[v + 1] - c.h_rowptr[v]) + (c.h_cscptr[v + 1] - c.h_cscptr[v]);
        if (k > 1024) {          // move.cu HUGE_THR
            c.h_huge.push_back(v);
            kmax_big = std::max(kmax_big, k);
        } else if (k > 256) {    // move.cu: 64-thread groups up to 256 entries
            c.h_big.push_back(v);
        } else if (k > 128) {    // move.cu BIG_THR
            c.h_mid.push_back(v);
        }
        if (k > 128 && k <= 1024) {
            c.h_midbig.push_back(v);
        }
    }
    // allocation: one device arena (one cudaMalloc / cudaFree per context),
    // planned in a measuring pass and then carved ---------------------------
    // persistent single-kernel sparse rebuild for graphs whose multi-kernel
    // rebuild is launch-bound (params.sparse_coop)
    c.coop_ok = c.prm.sparse_coop != 0 && (long long)E <= GSAP_COOP_MAX_E;
    const size_t Vs = (size_t)V, Es = (size_t)std::max(E, 1);
    const size_t VE = std::max(Vs, Es) + 1;
    const int P = c.prm.num_proposals;
    auto carve = [&](Arena &A) {
        c.rowptr = A.take<int>(Vs + 1);
        c.col = A.take<int>(Es);
        if (c.weighted) {
            c.wgt = A.take<int>(Es);
            c.cscwgt = A.take<int>(Es);
        }
        c.cscptr = A.take<int>(Vs + 1);
        c.cscsrc = A.take<int>(Es);
        c.esrc = A.take<int>(Es);
        c.kout = A.take<int>(Vs);
        c.kin = A.take<int>(Vs);
        c.selfw = A.take<int>(Vs);
        if (!c.h_big.empty()) c.big = A.take<int>(c.h_big.size());
        if (!c.h_mid.empty()) c.mid = A.take<int>(c.h_mid.size());
        if (!c.h_midbig.empty()) c.midbig = A.take<int>(c.h_midbig.size());
        if (!c.h_huge.empty()) {
            c.huge = A.take<int>(c.h_huge.size());
            const int log2cap = std::max(log2_ceil_h(2LL * std::min(kmax_big, V)), 5);
            if ((1 << log2cap) > 2048) {
                c.big_table_slots = (size_t)296 << log2cap;
                c.big_tables = A.take<int>(c.big_table_slots * 4);
            }
        }
        c.b = A.take<int>(Vs);
        {   // dense regime iff B^2 <= max(8 E, 2^24) (density >= 1/8, or M small): experiments may
            // override the multiplier (GSAP_DENSE_EMULT) and the floor (GSAP_DENSE_FLOOR_LOG2)
            int fl = 24, em = 8;
            if (const char *e = getenv("GSAP_DENSE_FLOOR_LOG2")) fl = std::max(16, std::min(29, atoi(e)));
            if (const char *e = getenv("GSAP_DENSE_EMULT")) em = std::max(1, std::min(64, atoi(e)));
            c.dense_cap = std::min<size_t>(std::max<size_t>((size_t)em * (size_t)E, (size_t)1 << fl), (size_t)1 << 29);
        }
        c.dense_cap = std::min<size_t>(c.dense_cap, Vs * Vs);
        if (c.prm.dense_max_B > 0)
            c.dense_cap = std::min<size_t>(c.dense_cap, (size_t)c.prm.dense_max_B * (size_t)c.prm.dense_max_B);
        // the lines of M: nnz <= E (sparse, compact or padded by degree) or B^2
        // (dense regime above SMALL_MAX_B: padded, line x at x B)
        const size_t Ls = std::max(Es, c.dense_cap);
        c.bm_rowptr = A.take<int>(Vs + 1);
        c.bm_colptr = A.take<int>(Vs + 1);
        c.bm_col = A.take<int>(Ls);
        c.bm_cnt = A.take<int>(Ls);
        c.bm_cum = A.take<int>(Ls);
        c.bm_row = A.take<int>(Ls);
        c.bm_ccnt = A.take<int>(Ls);
        c.bm_ccum = A.take<int>(Ls);
        c.dout = A.take<int>(Vs);
        c.din = A.take<int>(Vs);
        c.bm_rowend = A.take<int>(Vs);
        c.bm_colend = A.take<int>(Vs);
        c.d_nnz = A.take<int>(1);
        c.line_dirty = A.take<unsigned char>(2 * Vs);
        c.dl_arrive = A.take<unsigned>(1);
        c.dense = A.take<int>(c.dense_cap);
        c.rcp = A.take<double>(Vs);
        c.ft = A.take<double2>(FT_N);
        c.denseT = A.take<int>(c.dense_cap);
        c.keys0 = A.take<unsigned long long>(Es);
        c.keys1 = A.take<unsigned long long>(Es);
        c.vals64a = A.take<unsigned long long>(Es);
        c.vals64b = A.take<unsigned long long>(Es);
        c.ukeys0 = A.take<unsigned>(Es);
        c.ukeys1 = A.take<unsigned>(Es);
        c.wa = A.take<int>(VE);
        c.wb = A.take<int>(VE);
        c.flags = A.take<int>(VE);
        c.pos = A.take<int>(VE);
        c.tmpi = A.take<int>(VE);
        c.rownnz = A.take<int>(Vs + 1);
        c.seg_len = A.take<int>(Vs + 1);
        c.seg_cur = A.take<int>(Vs + 1);
        c.seg_nnz = A.take<int>(Vs + 1);
        c.seg_listW = A.take<int>(Vs + 1);
        c.seg_listC = A.take<int>(Vs + 1);
        c.seg_listM = A.take<int>(Vs + 1);
        c.seg_ctr = A.take<int>(8);
        c.xl_keys = A.take<unsigned long long>(2 * Es);
        c.xl_hp = A.take<int>(2 * Es);
        // the column side of both sparse rebuilds (persistent: its line scratch;
        // multi-kernel: everything, the two sides run concurrently)
        c.seg2_len = A.take<int>(Vs + 1);
        c.seg2_cur = A.take<int>(Vs + 1);
        c.seg2_nnz = A.take<int>(Vs + 1);
        c.seg2_listC = A.take<int>(Vs + 1);
        c.seg2_listW = A.take<int>(Vs + 1);
        c.seg2_listM = A.take<int>(Vs + 1);
        c.seg2_ctr = A.take<int>(8);
        c.xl2_keys = A.take<unsigned long long>(2 * Es);
        c.xl2_hp = A.take<int>(2 * Es);
        c.coop_bar = A.take<unsigned>(2);
        if (c.prm.dense_coop) c.small_acc = A.take<int>((size_t)SMALL_MAX_B * SMALL_MAX_B);
        const size_t tiles = (VE + 4095) / 4096 + 1;
        c.counts_cap = 256 * tiles;
        c.counts = A.take<int>(c.counts_cap);
        c.scan_tmp_cap = std::max(c.counts_cap, VE) / 4096 + 16;
        c.scan_tmp = A.take<int>(c.scan_tmp_cap);
        c.scan_tmp2 = A.take<int>(c.scan_tmp_cap);
        // per-batch / per-phase buffers, padded for the rank-blocked all-gathers
        const size_t pad = 65536;
        c.s = A.take<int>(std::max(Vs * (size_t)P, Vs + pad));
        c.dS = A.take<double>(std::max(Vs * (size_t)P, Vs + pad));
        c.H = A.take<double>(Vs + pad);
        c.acc = A.take<unsigned char>(Vs + pad);
        c.best = A.take<int>(Vs + pad);
        c.dSbest = A.take<double>(Vs + pad);
        // >= the MDL extent (max(E, B), or B^2 padded dense) / MDL_CHUNK, V / APPLY_CHUNK + ranks
        c.partials = A.take<double>(std::max(VE, c.dense_cap) / 512 + 1024);
        c.bpart = A.take<double>(Vs / 1024 + 2 * (size_t)std::max(1, c.prm.num_batches) + 16);
        c.scal = A.take<double>(8);
        c.scal_i = A.take<int>(8);
        c.n_eval = A.take<unsigned long long>(1);
        if (c.prm.proposal_mode == 1) c.mt = A.take<int>(Vs);
        c.dnnz_r = A.take<int>(Vs + 1);
        c.dnnz_c = A.take<int>(Vs + 1);
        // the move log: N2 (dense regime) and the neighbour-block cache's updates
        c.oldb = A.take<int>(Vs);
        c.moved = A.take<int>(Vs);
        c.movedb = A.take<int>(Vs);
        c.moved_cnt = A.take<int>(1);
        if (E > 0) {
            c.nbo = A.take<int>(Es);
            c.nbi = A.take<int>(Es);
            c.csc2csr = A.take<int>(Es);
            c.csr2csc = A.take<int>(Es);
        }
        c.Dh = A.take<double>((size_t)c.prm.max_nodal_itr + 1);
        if (c.prm.move_sorted) {
            c.mv_cnt = A.take<int>(2 * Vs + 2);
            c.mv_perm = A.take<int>(2 * Vs);
            c.mv_part = A.take<double>(3 * Vs);
            c.mv_scan_tmp = A.take<int>((2 * Vs + 4095) / 4096 + 16);
        }
        c.d_itr = A.take<unsigned>(1);
        c.skey0 = A.take<unsigned long long>(Vs);
        c.skey1 = A.take<unsigned long long>(Vs);
        c.sval0 = A.take<int>(Vs);
        c.sval1 = A.take<int>(Vs);
        c.sel_rank = A.take<int>(Vs);
        c.nxt0 = A.take<int>(Vs);
        c.nxt1 = A.take<int>(Vs);
        c.mx0 = A.take<int>(Vs);
        c.mx1 = A.take<int>(Vs);
        c.oncyc = A.take<int>(Vs);
        c.label = A.take<int>(Vs);
        c.present = A.take<int>(Vs + 1);
        for (int i = 0; i < 3; ++i) c.slot_b[i] = A.take<int>(Vs);
    };
    {
        Arena measure;
        carve(measure);
        void *base = nullptr;
        size_t got = 0;
        base = arena_take(c.dev, measure.off, &got);
        const cudaError_t e = base ? cudaSuccess : cudaMalloc(&base, measure.off);
        if (!got) got = measure.off;
        if (e == cudaErrorMemoryAllocation) {
            cudaGetLastError();
            throw Error{GSAP_ENOMEM, "cudaMalloc of the context arena failed"};
        }
        GSAP_CUDA(e);
        c.arena = base;
        c.arena_bytes = got;
        Arena cut;
        cut.base = (char *)base;
        carve(cut);
    }
    mark("arena");
    {   // f-table: f(m) = m ln m in long double, split into double hi + double lo (once per process)
        static std::vector<double2> ft;
        static std::once_flag once;
        std::call_once(once, [] {
            ft.resize(FT_N);
            for (int m = 0; m < FT_N; ++m) {
                const long double f = m > 0 ? (long double)m * logl((long double)m) : 0.0L;
                ft[m].x = (double)f;
                ft[m].y = (double)(f - (long double)ft[m].x);
            }
        });
        GSAP_CUDA(cudaMemcpyAsync(c.ft, ft.data(), sizeof(double2) * FT_N, cudaMemcpyHostToDevice, c.stream));
    }
    GSAP_CUDA(cudaMemsetAsync(c.coop_bar, 0, 2 * sizeof(unsigned), c.stream));
    GSAP_CUDA(cudaMemsetAsync(c.line_dirty, 0, 2 * (size_t)V, c.stream));
    GSAP_CUDA(cudaMemsetAsync(c.dl_arrive, 0, sizeof(unsigned), c.stream));
    if (c.small_acc)
        GSAP_CUDA(cudaMemsetAsync(c.small_acc, 0, sizeof(int) * SMALL_MAX_B * SMALL_MAX_B, c.stream));
    GSAP_CUDA(cudaMallocHost(&c.h_scal, 8 * sizeof(double)));
    GSAP_CUDA(cudaMallocHost(&c.h_int, 8 * sizeof(int)));
    mark("ftab+pinned");
    // upload ---------------------------------------------------------------
    GSAP_CUDA(cudaMemcpyAsync(c.rowptr, c.h_rowptr.data(), sizeof(int) * (Vs + 1), cudaMemcpyHostToDevice, c.stream));
    if (E) GSAP_CUDA(cudaMemcpyAsync(c.col, hc.data(), sizeof(int) * (size_t)E, cudaMemcpyHostToDevice, c.stream));
    if (c.weighted && E)
        GSAP_CUDA(cudaMemcpyAsync(c.wgt, hw.data(), sizeof(int) * (size_t)E, cudaMemcpyHostToDevice, c.stream));
    if (!c.h_big.empty())
        GSAP_CUDA(cudaMemcpyAsync(c.big, c.h_big.data(), sizeof(int) * c.h_big.size(), cudaMemcpyHostToDevice,
                                  c.stream));
    if (!c.h_midbig.empty())
        GSAP_CUDA(cudaMemcpyAsync(c.midbig, c.h_midbig.data(), sizeof(int) * c.h_midbig.size(),
                                  cudaMemcpyHostToDevice, c.stream));
    if (!c.h_mid.empty())
        GSAP_CUDA(cudaMemcpyAsync(c.mid, c.h_mid.data(), sizeof(int) * c.h_mid.size(), cudaMemcpyHostToDevice,
                                  c.stream));
    if (!c.h_huge.empty())
        GSAP_CUDA(cudaMemcpyAsync(c.huge, c.h_huge.data(), sizeof(int) * c.h_huge.size(),
                                  cudaMemcpyHostToDevice, c.stream));
    GSAP_CUDA(cudaMemsetAsync(c.scal, 0, 8 * sizeof(double), c.stream));
    GSAP_CUDA(cudaMemsetAsync(c.scal_i, 0, 8 * sizeof(int), c.stream));
    GSAP_CUDA(cudaMemsetAsync(c.n_eval, 0, sizeof(unsigned long long), c.stream));
    mark("upload");
    build_graph_device(c);
    mark("csc");
    // the singleton partition (P:61 2.1)
    std::vector<int> iota(Vs);
    for (int v = 0; v < V; ++v) iota[v] = v;
    GSAP_CUDA(cudaMemcpyAsync(c.b, iota.data(), sizeof(int) * Vs, cudaMemcpyHostToDevice, c.stream));
    c.B = V;
    b_changed(c);
    rebuild(c);
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    mark("rebuild");
}

// ------------------------------------------------------------- driver --
static void set_iota(Ctx &c) {
    std::vector<int> iota((size_t)c.V);
    for (int v = 0; v < c.V; ++v) iota[v] = v;
    GSAP_CUDA(cudaMemcpyAsync(c.b, iota.data(), sizeof(int) * (size_t)c.V, cudaMemcpyHostToDevice, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    c.B = c.V;
    b_changed(c);
}

static double mdl_now(Ctx &c) {
    return model_term(c.W, c.V, c.B, c.prm.model_term) + device_data_term(c);
}

// ranks the batches and merge phases are sliced over: the NCCL ranks, or the
// ranks one process emulates (params.sim_ranks: every slice computed here in
// rank order, the exchange skipped -- the sharded data path on one GPU)
static int ranks_of(const Ctx &c) { return c.nranks > 1 ? c.nranks : std::max(1, c.prm.sim_ranks); }

static void merge_phase(Ctx &c, uint32_t outer, int K, int *best_out, double *dSbest_out) {
    REQUIRE(c.B >= 2, GSAP_ESTATE, "a merge phase needs B >= 2");
    REQUIRE(K >= 0 && K <= c.B / 2, GSAP_EINVAL, "K must be in [0, B/2]");
    const int B = c.B;
    const int G = ranks_of(c);
    launch_fill_mt(c, TABLE_J, 0, outer, 0);   // N4 ablation only
    if (G == 1) {
        launch_merge_props(c, outer, 0, B, true, nullptr, nullptr, c.best, c.dSbest);
        c.st.n_merge_prop += (long long)B * c.prm.num_proposals;
    } else {
        // each rank proposes for its range of blocks (equal counts); the
        // winners (12 B per block) are all-gathered; every rank then runs the
        // identical selection and rebuild.  sim_ranks: all slices here, in order.
        std::vector<int> f(G), n(G);
        for (int g = 0; g < G; ++g) {
            int per;
            shard_slice(B, 1, G, g, &f[g], &n[g], &per);
        }
        const int g0 = c.nranks > 1 ? c.rank : 0, g1 = c.nranks > 1 ? c.rank + 1 : G;
        for (int g = g0; g < g1; ++g) {
            if (n[g] > 0) launch_merge_props(c, outer, f[g], n[g], true, nullptr, nullptr, c.best + f[g], c.dSbest + f[g]);
            c.st.n_merge_prop += (long long)n[g] * c.prm.num_proposals;
        }
        comm_allgatherv(c, c.best, f, n, 1);
        comm_allgatherv(c, c.dSbest, f, n, 2);
    }
    copy_out(c, best_out, c.best, sizeof(int) * (size_t)B);
    copy_out(c, dSbest_out, c.dSbest, sizeof(double) * (size_t)B);
    select_merges(c, c.best, c.dSbest, K, nullptr);
    rebuild(c);
}

// N2: the next rebuild may apply the batch's moves to the dense M of the
// previous one (the apply logs them); the sparse regime rebuilds in full
static void announce_batch(Ctx &c, int first, int count) {
    c.delta.first = first;
    c.delta.count = count;
    c.delta.acc = c.acc;
    c.delta.pending = c.prm.incremental != 0 && c.dense_mode && c.oldb != nullptr;
}

static void move_batch(Ctx &c, uint32_t outer, uint32_t itr, int first, int count, double *dsum) {
    c.batch_count = count;
    const int G = ranks_of(c);
    announce_batch(c, first, count);
    launch_fill_mt(c, TABLE_J | ((uint32_t)first & 0x3fffffffu), itr, outer, 1);   // N4 ablation only
    if (G == 1) {
        launch_move(c, MOVE_FUSED, outer, itr, first, count, c.s, c.dS, nullptr, c.acc);
        launch_apply(c, first, count, c.s, c.acc, c.dS, dsum, c.scal_i + 1, c.n_eval);
        rebuild(c);
        c.st.n_move_prop += count;
        return;
    }
    // the batch cut into G edge-balanced slices of whole APPLY_CHUNK_V chunks;
    // this rank evaluates its slice (sim_ranks: every slice, in order) and the
    // fixed-chunk dS partials of its accepted moves; ONE exchange step: the
    // slices' s, acc and partials all-gathered in place (contiguous, no
    // padding); then every rank applies the whole batch, sums the partials in
    // chunk order and rebuilds -- the same operations in the same order as
    // G = 1, so the trajectory is bit-identical for any G.
    std::vector<int> f, n;
    shard_plan(c, first, count, G, f, n);
    const int CH = APPLY_CHUNK_V;
    const int g0 = c.nranks > 1 ? c.rank : 0, g1 = c.nranks > 1 ? c.rank + 1 : G;
    for (int g = g0; g < g1; ++g) {
        if (n[g] <= 0) continue;
        launch_move(c, MOVE_FUSED, outer, itr, first + f[g], n[g], c.s + f[g], c.dS + f[g], nullptr, c.acc + f[g]);
        launch_partials(c, first + f[g], n[g], c.s + f[g], c.acc + f[g], c.dS + f[g], c.partials + f[g] / CH);
        c.st.n_move_prop += n[g];
    }
    if (c.nranks > 1) {
        std::vector<int> pf(G), pn(G);
        for (int g = 0; g < G; ++g) {
            pf[g] = f[g] / CH;
            pn[g] = (n[g] + CH - 1) / CH;
        }
        comm_allgatherv(c, c.s, f, n, 1);
        comm_allgatherv(c, c.acc, f, n, 0);
        comm_allgatherv(c, c.partials, pf, pn, 2);
    }
    const int chunks = (count + CH - 1) / CH;
    launch_apply_gathered(c, first, count, c.s, c.acc, c.partials, chunks, dsum, c.scal_i + 1, c.n_eval);
    rebuild(c);
}

static bool converged(Ctx &c, const std::vector<double> &D, int itr, double S, double thresh) {
    const int w = c.prm.window;
    if (itr < w - 1) return false;
    const double mdl = model_term(c.W, c.V, c.B, c.prm.model_term) + S;
    double sum = 0.0;
    int n = 0;
    for (int j = itr - w + 1; j < itr; ++j) {
        sum += D[j];
        ++n;
    }
    const double mean = n ? sum / n : 0.0;
    return -mean < thresh * mdl;
}

// MCMC phase with every iteration (num_batches x (move + apply + rebuild) +
// the MDL reduction) captured once into a CUDA graph; one graph launch, one
// 16-byte D2H and one synchronisation per iteration.
static int mcmc_phase_graph(Ctx &c, uint32_t outer, double thresh, std::vector<double> *D_out) {
    const int V = c.V, nb = c.prm.num_batches;
    const int bs = (V + nb - 1) / nb;
    const int nch = (bs + APPLY_CHUNK_V - 1) / APPLY_CHUNK_V;   // dS chunk partials per full batch
    DsumSpec ds{c.bpart, 0, nch, nch, 0};
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
    const long long l0 = c.launches;
    const auto tcs = std::chrono::steady_clock::now();
    GSAP_CUDA(cudaStreamBeginCapture(c.stream, cudaStreamCaptureModeThreadLocal));
    c.capturing = true;
    try {
        GSAP_CUDA(cudaMemsetAsync(c.scal, 0, sizeof(double), c.stream));
        for (int k = 0; k < nb; ++k) {
            const int first = k * bs, last = std::min(V, first + bs);
            if (first >= last) continue;
            c.batch_count = last - first;
            announce_batch(c, first, last - first);
            launch_fill_mt(c, TABLE_J | ((uint32_t)first & 0x3fffffffu), 0, outer, 1, c.d_itr);   // N4 only
            launch_move(c, MOVE_FUSED, outer, 0, first, last - first, c.s, c.dS, nullptr, c.acc, c.d_itr);
            launch_apply_deferred(c, first, last - first, c.s, c.acc, c.dS, c.bpart + (size_t)k * ds.stride,
                                  c.scal_i + 1, c.n_eval);
            rebuild(c);
            ds.nbat = k + 1;
            ds.nch_last = (last - first + APPLY_CHUNK_V - 1) / APPLY_CHUNK_V;
        }
        nb_join(c);   // no side-stream work may stay unjoined in a capture
        launch_data_term(c, &ds);   // the MDL and the iteration's dS sum (c.scal[1], c.scal[0])
    } catch (...) {
        c.capturing = false;
        cudaStreamEndCapture(c.stream, &graph);
        if (graph) cudaGraphDestroy(graph);
        graph_release_events(c);
        throw;
    }
    c.capturing = false;
    GSAP_CUDA(cudaStreamEndCapture(c.stream, &graph));
    const long long kernels = c.launches - l0;
    c.launches = l0;
    const auto tc0 = std::chrono::steady_clock::now();
    exec = mcmc_exec_for(c, graph, 1);
    const auto tc1 = std::chrono::steady_clock::now();
    std::vector<double> D((size_t)c.prm.max_nodal_itr + 1, 0.0);
    int ran = 0;
    try {
        for (int itr = 0; itr < c.prm.max_nodal_itr; ++itr) {
            c.h_int[2] = itr;
            GSAP_CUDA(cudaMemcpyAsync(c.d_itr, c.h_int + 2, sizeof(unsigned), cudaMemcpyHostToDevice, c.stream));
            GSAP_CUDA(cudaGraphLaunch(exec, c.stream));
            GSAP_CUDA(cudaMemcpyAsync(c.h_scal, c.scal, 2 * sizeof(double), cudaMemcpyDeviceToHost, c.stream));
            GSAP_CUDA(cudaStreamSynchronize(c.stream));
            c.launches += kernels;
            c.st.n_move_prop += V;
            graph_account(c);
            D[itr] = c.h_scal[0];
            ran = itr + 1;
            if (converged(c, D, itr, c.h_scal[1], thresh)) break;
        }
    } catch (...) {
        drop_mcmc_exec(c);
        cudaGraphDestroy(graph);
        graph_release_events(c);
        throw;
    }
    GSAP_CUDA(cudaGraphDestroy(graph));
    graph_release_events(c);
    if (D_out) D_out->assign(D.begin(), D.begin() + ran);
    if (getenv("GSAP_TIMING")) {
        const auto tc2 = std::chrono::steady_clock::now();
        fprintf(stderr, "[gsap] mcmc B=%d kernels/itr=%lld capture %.3f ms instantiate %.3f ms %d itrs %.3f ms\n", c.B,
                kernels, std::chrono::duration<double, std::milli>(tc0 - tcs).count(),
                std::chrono::duration<double, std::milli>(tc1 - tc0).count(), ran,
                std::chrono::duration<double, std::milli>(tc2 - tc1).count());
    }
    return ran;
}

// End of one MCMC iteration inside the device-side loop (R:O.8, R:Z19): D[itr]
// = the iteration's sum of accepted dS, the GraphChallenge convergence test on
// the device -- the same double operations in the same order as converged()
// on the host -- and the while-condition of the enclosing conditional node.
__global__ void k_mcmc_step(cudaGraphConditionalHandle h, unsigned *d_itr, double *scal, double *Dh, int max_itr,
                            int w, double model, double thresh) {
    const int itr = (int)*d_itr;
    Dh[itr] = scal[0];
    scal[0] = 0.0;
    bool stop = itr + 1 >= max_itr;
    if (!stop && itr >= w - 1) {
        double sum = 0.0;
        int n = 0;
        for (int j = itr - w + 1; j < itr; ++j) {
            sum += Dh[j];
            ++n;
        }
        const double mean = n ? sum / n : 0.0;
        const double mdl = model + scal[1];
        stop = -mean < thresh * mdl;
    }
    *d_itr = (unsigned)(itr + 1);
    cudaGraphSetConditional(h, stop ? 0u : 1u);
}

// The whole MCMC phase as ONE graph launch: a conditional WHILE node whose
// body is one iteration (num_batches x (move + apply + rebuild), the MDL
// reduction, k_mcmc_step); the loop runs on the device until the
// convergence test or max_nodal_itr stops it -- no host round trip per
// iteration (N1, P:385 5).  Event nodes are not allowed in conditional
// bodies, so profile = 1 uses mcmc_phase_graph.
static int mcmc_phase_device_loop(Ctx &c, uint32_t outer, double thresh, std::vector<double> *D_out) {
    const int V = c.V, nb = c.prm.num_batches;
    const int bs = (V + nb - 1) / nb;
    const int nch = (bs + APPLY_CHUNK_V - 1) / APPLY_CHUNK_V;   // dS chunk partials per full batch
    DsumSpec ds{c.bpart, 0, nch, nch, 0};
    const long long l0 = c.launches;
    const auto tcs = std::chrono::steady_clock::now();
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
    GSAP_CUDA(cudaGraphCreate(&graph, 0));
    try {
        cudaGraphConditionalHandle h;
        GSAP_CUDA(cudaGraphConditionalHandleCreate(&h, graph, 1u, cudaGraphCondAssignDefault));
        cudaGraphNodeParams np = {};
        np.type = cudaGraphNodeTypeConditional;
        np.conditional.handle = h;
        np.conditional.type = cudaGraphCondTypeWhile;
        np.conditional.size = 1;
        cudaGraphNode_t node;
        GSAP_CUDA(cudaGraphAddNode(&node, graph, nullptr, 0, &np));
        cudaGraph_t body = np.conditional.phGraph_out[0];
        GSAP_CUDA(cudaStreamBeginCaptureToGraph(c.stream, body, nullptr, nullptr, 0,
                                                cudaStreamCaptureModeThreadLocal));
        c.capturing = true;
        try {
            for (int k = 0; k < nb; ++k) {
                const int first = k * bs, last = std::min(V, first + bs);
                if (first >= last) continue;
                c.batch_count = last - first;
            announce_batch(c, first, last - first);
            launch_fill_mt(c, TABLE_J | ((uint32_t)first & 0x3fffffffu), 0, outer, 1, c.d_itr);   // N4 only
            launch_move(c, MOVE_FUSED, outer, 0, first, last - first, c.s, c.dS, nullptr, c.acc, c.d_itr);
                launch_apply_deferred(c, first, last - first, c.s, c.acc, c.dS, c.bpart + (size_t)k * ds.stride,
                                      c.scal_i + 1, c.n_eval);
                rebuild(c);
                ds.nbat = k + 1;
                ds.nch_last = (last - first + APPLY_CHUNK_V - 1) / APPLY_CHUNK_V;
            }
            nb_join(c);   // no side-stream work may stay unjoined in a capture
            launch_data_term(c, &ds);   // the MDL and the iteration's dS sum (c.scal[1], c.scal[0])
            const double model = model_term(c.W, c.V, c.B, c.prm.model_term);
            k_mcmc_step<<<1, 1, 0, c.stream>>>(h, c.d_itr, c.scal, c.Dh, c.prm.max_nodal_itr, c.prm.window, model,
                                              thresh);
            GSAP_CHECK_LAUNCH();
            ++c.launches;
        } catch (...) {
            c.capturing = false;
            cudaGraph_t g2 = nullptr;
            cudaStreamEndCapture(c.stream, &g2);
            throw;
        }
        c.capturing = false;
        GSAP_CUDA(cudaStreamEndCapture(c.stream, &body));
        const long long kernels = c.launches - l0;
        c.launches = l0;
        const auto tc0 = std::chrono::steady_clock::now();
        exec = mcmc_exec_for(c, graph, 2);
        const auto tc1 = std::chrono::steady_clock::now();
        GSAP_CUDA(cudaMemsetAsync(c.scal, 0, sizeof(double), c.stream));
        GSAP_CUDA(cudaMemsetAsync(c.d_itr, 0, sizeof(unsigned), c.stream));
        GSAP_CUDA(cudaGraphLaunch(exec, c.stream));
        GSAP_CUDA(cudaMemcpyAsync(c.h_int + 2, c.d_itr, sizeof(unsigned), cudaMemcpyDeviceToHost, c.stream));
        GSAP_CUDA(cudaStreamSynchronize(c.stream));
        const int ran = c.h_int[2];
        if (D_out) {
            D_out->resize((size_t)ran);
            if (ran)
                GSAP_CUDA(cudaMemcpy(D_out->data(), c.Dh, sizeof(double) * (size_t)ran, cudaMemcpyDeviceToHost));
        }
        c.launches += kernels * ran;
        c.st.n_move_prop += (long long)V * ran;
        GSAP_CUDA(cudaGraphDestroy(graph));
        if (getenv("GSAP_TIMING")) {
            const auto tc2 = std::chrono::steady_clock::now();
            fprintf(stderr, "[gsap] mcmc(device loop) B=%d kernels/itr=%lld capture %.3f ms instantiate %.3f ms "
                    "%d itrs %.3f ms\n", c.B, kernels, std::chrono::duration<double, std::milli>(tc0 - tcs).count(),
                    std::chrono::duration<double, std::milli>(tc1 - tc0).count(), ran,
                    std::chrono::duration<double, std::milli>(tc2 - tc1).count());
        }
        return ran;
    } catch (...) {
        if (exec) drop_mcmc_exec(c);
        cudaGraphDestroy(graph);
        throw;
    }
}

// returns the number of MCMC iterations run (O.8); D_out (nullable): D[itr]
static int mcmc_phase(Ctx &c, uint32_t outer, double thresh, std::vector<double> *D_out = nullptr) {
    if (c.prm.cuda_graphs == 2 && !c.prm.profile && c.nranks == 1)
        return mcmc_phase_device_loop(c, outer, thresh, D_out);
    if (c.prm.cuda_graphs) return mcmc_phase_graph(c, outer, thresh, D_out);
    const int V = c.V, nb = c.prm.num_batches, w = c.prm.window;
    const int bs = (V + nb - 1) / nb;
    std::vector<double> D((size_t)c.prm.max_nodal_itr + 1, 0.0);
    int ran = 0;
    for (int itr = 0; itr < c.prm.max_nodal_itr; ++itr) {
        GSAP_CUDA(cudaMemsetAsync(c.Dh + itr, 0, sizeof(double), c.stream));
        for (int k = 0; k < nb; ++k) {
            const int first = k * bs, last = std::min(V, first + bs);
            if (first >= last) continue;
            move_batch(c, outer, (uint32_t)itr, first, last - first, c.Dh + itr);
        }
        ran = itr + 1;
        if (itr >= w - 1) {
            launch_data_term(c);
            GSAP_CUDA(cudaMemcpyAsync(c.h_scal + 1, c.scal + 1, sizeof(double), cudaMemcpyDeviceToHost, c.stream));
            GSAP_CUDA(cudaMemcpyAsync(D.data(), c.Dh, sizeof(double) * (size_t)(itr + 1), cudaMemcpyDeviceToHost,
                                      c.stream));
            GSAP_CUDA(cudaStreamSynchronize(c.stream));
            if (converged(c, D, itr, c.h_scal[1], thresh)) break;
        }
    }
    if (D_out) {
        D_out->resize((size_t)ran);
        if (ran) GSAP_CUDA(cudaMemcpy(D_out->data(), c.Dh, sizeof(double) * (size_t)ran, cudaMemcpyDeviceToHost));
    }
    return ran;
}

namespace {
// golden-section bracket over (b, B, MDL), slot 1 = best (GraphChallenge's
// prepare_for_partition_on_next_num_blocks; R:Z21).  Returns true when done.
struct Bracket {
    int B[3] = {0, 0, 0};
    double S[3] = {INFINITY, INFINITY, INFINITY};
};

bool bracket_update(Ctx &c, Bracket &br, int B, double S, int *K, int *restart) {
    auto copy_slot = [&](int dst, const int *src) {
        GSAP_CUDA(cudaMemcpyAsync(c.slot_b[dst], src, sizeof(int) * (size_t)c.V, cudaMemcpyDeviceToDevice,
                                  c.stream));
    };
    int idx;
    if (S <= br.S[1]) {
        idx = br.B[1] > B ? 0 : 2;
        copy_slot(idx, c.slot_b[1]);
        br.B[idx] = br.B[1];
        br.S[idx] = br.S[1];
        idx = 1;
    } else {
        idx = br.B[1] > B ? 2 : 0;
    }
    copy_slot(idx, c.b);
    br.B[idx] = B;
    br.S[idx] = S;
    if (br.S[2] == INFINITY) {
        *K = (int)((double)B * c.prm.reduction_rate);
        *restart = 1;
        return *K == 0;
    }
    if (br.B[0] - br.B[2] == 2) return true;
    const int i = (br.B[0] - br.B[1]) >= (br.B[1] - br.B[2]) ? 0 : 1;
    const int next = br.B[i + 1] + (int)nearbyint((double)(br.B[i] - br.B[i + 1]) * 0.618);
    *K = br.B[i] - next;
    *restart = i;
    return *K <= 0;
}
}  // namespace

static void run_impl(Ctx &c, int32_t *bmap_out, int32_t *B_out, double *mdl_out, double *trace, int trace_cap,
                     int32_t *rounds_out) {
    const auto t0 = std::chrono::steady_clock::now();
    GSAP_CUDA(cudaMemsetAsync(c.scal_i + 1, 0, sizeof(int), c.stream));
    set_iota(c);
    rebuild(c);
    Bracket br;
    int K = (int)((double)c.B * c.prm.reduction_rate);
    uint32_t outer = 0;
    int rounds = 0;
    bool done = false;
    if (K == 0) {
        br.S[1] = mdl_now(c);
        br.B[1] = c.B;
        GSAP_CUDA(cudaMemcpyAsync(c.slot_b[1], c.b, sizeof(int) * (size_t)c.V, cudaMemcpyDeviceToDevice, c.stream));
        done = true;
    }
    double t_merge = 0, t_move = 0, t_mdl = 0;
    while (!done && rounds < c.prm.max_rounds) {
        const bool bracket = br.S[2] != INFINITY;
        int acc_before = 0;
        double ms0[3] = {0.0, 0.0, 0.0};
        if (trace && rounds < trace_cap) {
            kc_resolve(c, c.k_move);
            kc_resolve(c, c.k_rebuild);
            kc_resolve(c, c.k_merge);
            ms0[0] = c.k_move.ms;
            ms0[1] = c.k_rebuild.ms;
            ms0[2] = c.k_merge.ms;
            GSAP_CUDA(cudaMemcpyAsync(c.h_int + 3, c.scal_i + 1, sizeof(int), cudaMemcpyDeviceToHost, c.stream));
            GSAP_CUDA(cudaStreamSynchronize(c.stream));
            acc_before = c.h_int[3];
        }
        auto ta = std::chrono::steady_clock::now();
        const int B_start = c.B, K_round = K;
        merge_phase(c, outer, K, nullptr, nullptr);
        const int B = c.B;
        auto tb = std::chrono::steady_clock::now();
        const int itrs = mcmc_phase(c, outer, bracket ? c.prm.thresh2 : c.prm.thresh1);
        auto tc = std::chrono::steady_clock::now();
        const double S = mdl_now(c);
        auto td = std::chrono::steady_clock::now();
        if (getenv("GSAP_TIMING"))
            fprintf(stderr, "[gsap] round %d B=%d merge %.3f ms mcmc %.3f ms mdl %.3f ms\n", rounds, B,
                    std::chrono::duration<double, std::milli>(tb - ta).count(),
                    std::chrono::duration<double, std::milli>(tc - tb).count(),
                    std::chrono::duration<double, std::milli>(td - tc).count());
        t_merge += std::chrono::duration<double>(tb - ta).count();
        t_move += std::chrono::duration<double>(tc - tb).count();
        t_mdl += std::chrono::duration<double>(td - tc).count();
        if (trace && rounds < trace_cap) {
            GSAP_CUDA(cudaMemcpyAsync(c.h_int + 3, c.scal_i + 1, sizeof(int), cudaMemcpyDeviceToHost, c.stream));
            GSAP_CUDA(cudaStreamSynchronize(c.stream));
            double *row = trace + (size_t)GSAP_TRACE_COLS * rounds;
            row[0] = (double)outer;
            row[1] = (double)B;
            row[2] = (double)itrs;
            row[3] = S;
            row[4] = std::chrono::duration<double>(td - ta).count();
            row[5] = (double)(c.h_int[3] - acc_before);
            // device ms of the kernel classes in this round (profile = 1)
            kc_resolve(c, c.k_move);
            kc_resolve(c, c.k_rebuild);
            kc_resolve(c, c.k_merge);
            row[6] = c.k_move.ms - ms0[0];
            row[7] = c.k_rebuild.ms - ms0[1];
            row[8] = c.k_merge.ms - ms0[2];
            row[9] = bracket ? c.prm.thresh2 : c.prm.thresh1;
            row[10] = (double)B_start;
            row[11] = (double)K_round;
        }
        c.st.mcmc_itr_total += itrs;
        ++rounds;
        int restart = 1;
        if (bracket_update(c, br, B, S, &K, &restart)) break;
        GSAP_CUDA(cudaMemcpyAsync(c.b, c.slot_b[restart], sizeof(int) * (size_t)c.V, cudaMemcpyDeviceToDevice,
                                  c.stream));
        c.B = br.B[restart];
        b_changed(c);
        rebuild(c);
        ++outer;
    }
    if (br.B[1] == 0) {   // no round ran (max_rounds = 0): the answer is the current partition
        br.B[1] = c.B;
        br.S[1] = mdl_now(c);
        GSAP_CUDA(cudaMemcpyAsync(c.slot_b[1], c.b, sizeof(int) * (size_t)c.V, cudaMemcpyDeviceToDevice, c.stream));
    }
    // the answer: slot 1
    GSAP_CUDA(cudaMemcpyAsync(c.b, c.slot_b[1], sizeof(int) * (size_t)c.V, cudaMemcpyDeviceToDevice, c.stream));
    c.B = br.B[1];
    b_changed(c);
    rebuild(c);
    copy_out(c, bmap_out, c.b, sizeof(int) * (size_t)c.V);
    GSAP_CUDA(cudaMemcpyAsync(c.h_int + 1, c.scal_i + 1, sizeof(int), cudaMemcpyDeviceToHost, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    c.st.n_move_acc += c.h_int[1];
    if (B_out) *B_out = c.B;
    if (mdl_out) *mdl_out = br.S[1];
    if (rounds_out) *rounds_out = rounds;
    c.st.rounds += rounds;
    c.st.B_final = c.B;
    c.st.t_merge += t_merge;
    c.st.t_move += t_move;
    c.st.t_mdl += t_mdl;
    c.st.t_total += std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
}

static void fill_stats(Ctx &c, gsap_stats *out) {
    for (KClass *k : {&c.k_move, &c.k_rebuild, &c.k_merge, &c.k_mdl, &c.k_comm, &c.k_groups, &c.k_warps})
        kc_resolve(c, *k);
    if (getenv("GSAP_TIMING") && (c.k_groups.launches || c.k_warps.launches))
        fprintf(stderr, "[gsap] MOVE roles (profile, outside graphs): group role %lld launches %.3f ms, "
                "warp role %lld launches %.3f ms\n", c.k_groups.launches, c.k_groups.ms, c.k_warps.launches,
                c.k_warps.ms);
    gsap_stats s = c.st;
    unsigned long long ne = 0;
    GSAP_CUDA(cudaMemcpyAsync(&ne, c.n_eval, sizeof(ne), cudaMemcpyDeviceToHost, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    s.n_move_eval = (int64_t)ne;
    s.t_rebuild = c.k_rebuild.ms * 1e-3;
    s.t_comm = c.k_comm.ms * 1e-3;
    s.gpu_launches = c.launches;
    s.k_move_ms = c.k_move.ms;
    s.k_move_bytes = c.k_move.bytes;
    s.k_move_launches = c.k_move.launches;
    s.k_rebuild_ms = c.k_rebuild.ms;
    s.k_rebuild_bytes = c.k_rebuild.bytes;
    s.k_rebuild_launches = c.k_rebuild.launches;
    s.k_merge_ms = c.k_merge.ms;
    s.k_merge_bytes = c.k_merge.bytes;
    s.k_merge_launches = c.k_merge.launches;
    s.k_mdl_ms = c.k_mdl.ms;
    s.k_mdl_launches = c.k_mdl.launches;
    *out = s;
}

// ================================================================ C-ABI ===
extern "C" {

void gsap_default_params(gsap_params *p) {
    if (!p) return;
    memset(p, 0, sizeof(*p));
    p->seed = 0x5B9D2024ULL;
    p->beta = 3.0;
    p->reduction_rate = 0.4;
    p->num_proposals = 10;
    p->max_nodal_itr = 100;
    p->thresh1 = 5e-4;
    p->thresh2 = 1e-4;
    p->window = 3;
    p->num_batches = 4;
    p->model_term = 0;
    p->max_rounds = 500;
    p->profile = 0;
    p->cuda_graphs = 2;
    p->dense_max_B = 0;
    p->sparse_coop = 1;
    p->dense_coop = 1;
    p->sel_small = 1;
    p->move_sorted = 1;
    p->sim_ranks = 0;
    p->incremental = 1;
    p->proposal_mode = 0;
    p->line_sort = 1;
}

const char *gsap_last_error(void) { return g_err.c_str(); }

gsap_status gsap_create(int32_t V, const int64_t *rowptr, const int32_t *col, const int32_t *wgt,
                        const gsap_params *params, const gsap_dist *dist, void *stream, gsap_ctx **out) {
    API_TRY
    REQUIRE(out, GSAP_EINVAL, "out is NULL");
    *out = nullptr;
    gsap_ctx *h = new gsap_ctx();
    try {
        create_impl(h->c, V, rowptr, col, wgt, params, dist, stream);
    } catch (...) {
        free_ctx(h->c);
        delete h;
        throw;
    }
    *out = h;
    API_CATCH
}

void gsap_destroy(gsap_ctx *ctx) {
    if (!ctx) return;
    if (ctx->c.stream) cudaStreamSynchronize(ctx->c.stream);
    free_ctx(ctx->c);
    delete ctx;
}

gsap_status gsap_set_partition(gsap_ctx *ctx, const int32_t *b, int32_t B) {
    API_TRY
    REQUIRE(ctx && b, GSAP_EINVAL, "NULL argument");
    Ctx &c = ctx->c;
    REQUIRE(B >= 1 && B <= c.V, GSAP_EINVAL, "B must be in [1, V]");
    if (!is_dev(b)) {
        for (int v = 0; v < c.V; ++v) REQUIRE(b[v] >= 0 && b[v] < B, GSAP_EINVAL, "b[v] out of [0, B)");
    } else {
        REQUIRE(device_ids_ok(c, c.V, b, nullptr, B, false), GSAP_EINVAL, "b[v] out of [0, B)");
    }
    GSAP_CUDA(cudaMemcpyAsync(c.b, b, sizeof(int) * (size_t)c.V, cudaMemcpyDefault, c.stream));
    c.B = B;
    b_changed(c);
    rebuild(c);
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    API_CATCH
}

gsap_status gsap_get_partition(gsap_ctx *ctx, int32_t *b_out, int32_t *B_out) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    copy_out(ctx->c, b_out, ctx->c.b, sizeof(int) * (size_t)ctx->c.V);
    if (B_out) *B_out = ctx->c.B;
    API_CATCH
}

gsap_status gsap_update_blockmodel(gsap_ctx *ctx) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    rebuild(ctx->c);
    API_CATCH
}

gsap_status gsap_propose(gsap_ctx *ctx, gsap_phase phase, uint32_t outer, uint32_t itr, int32_t first,
                         int32_t count, int32_t *s_out) {
    API_TRY
    REQUIRE(ctx && s_out, GSAP_EINVAL, "NULL argument");
    Ctx &c = ctx->c;
    const int n = phase == GSAP_MOVE ? c.V : c.B;
    REQUIRE(first >= 0 && count >= 0 && (long long)first + count <= n, GSAP_EINVAL, "range out of bounds");
    if (count == 0) return GSAP_OK;
    if (phase == GSAP_MOVE) {
        launch_fill_mt(c, TABLE_J | ((uint32_t)first & 0x3fffffffu), itr, outer, 1);   // N4: table keyed by `first`
        launch_move(c, MOVE_PROPOSE, outer, itr, first, count, c.s, nullptr, nullptr, nullptr);
        copy_out(c, s_out, c.s, sizeof(int) * (size_t)count);
    } else {
        REQUIRE(c.B >= 2, GSAP_ESTATE, "merge proposals need B >= 2");
        launch_fill_mt(c, TABLE_J, 0, outer, 0);   // N4
        launch_merge_props(c, outer, first, count, true, c.s, nullptr, nullptr, nullptr);
        copy_out(c, s_out, c.s, sizeof(int) * (size_t)count * c.prm.num_proposals);
    }
    API_CATCH
}

gsap_status gsap_delta_mdl(gsap_ctx *ctx, gsap_phase phase, uint32_t outer, uint32_t itr, int32_t first,
                           int32_t count, const int32_t *s, double *dS_out, double *H_out, uint8_t *acc_out) {
    API_TRY
    REQUIRE(ctx && s, GSAP_EINVAL, "NULL argument");
    Ctx &c = ctx->c;
    const int n = phase == GSAP_MOVE ? c.V : c.B;
    REQUIRE(first >= 0 && count >= 0 && (long long)first + count <= n, GSAP_EINVAL, "range out of bounds");
    if (count == 0) return GSAP_OK;
    if (phase == GSAP_MOVE) {
        const int *ds = stage_in(c, s, (size_t)count, c.s);
        launch_move(c, MOVE_DELTA, outer, itr, first, count, const_cast<int *>(ds), c.dS, c.H, c.acc);
        copy_out(c, dS_out, c.dS, sizeof(double) * (size_t)count);
        copy_out(c, H_out, c.H, sizeof(double) * (size_t)count);
        copy_out(c, acc_out, c.acc, (size_t)count);
    } else {
        REQUIRE(c.B >= 2, GSAP_ESTATE, "merge proposals need B >= 2");
        const size_t np = (size_t)count * c.prm.num_proposals;
        const int *ds = stage_in(c, s, np, c.s);
        launch_merge_props(c, outer, first, count, false, const_cast<int *>(ds), c.dS, nullptr, nullptr);
        copy_out(c, dS_out, c.dS, sizeof(double) * np);
    }
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    API_CATCH
}

gsap_status gsap_select_merges(gsap_ctx *ctx, const int32_t *best, const double *dS, int32_t K,
                               int32_t *label_out, int32_t *newB_out) {
    API_TRY
    REQUIRE(ctx && best && dS, GSAP_EINVAL, "NULL argument");
    Ctx &c = ctx->c;
    REQUIRE(c.B >= 2, GSAP_ESTATE, "selection needs B >= 2");
    REQUIRE(K >= 0 && K <= c.B / 2, GSAP_EINVAL, "K must be in [0, B/2]");
    const int B = c.B;
    if (!is_dev(best))
        for (int r = 0; r < B; ++r)
            REQUIRE(best[r] >= 0 && best[r] < B && best[r] != r, GSAP_EINVAL, "best[r] must be in [0,B), != r");
    else
        REQUIRE(device_ids_ok(c, B, best, nullptr, B, true), GSAP_EINVAL, "best[r] must be in [0,B), != r");
    const int *db = stage_in(c, best, (size_t)B, c.best);
    const double *dd = stage_in(c, dS, (size_t)B, c.dSbest);
    select_merges(c, db, dd, K, nullptr);
    copy_out(c, label_out, c.label, sizeof(int) * (size_t)B);
    rebuild(c);
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    if (newB_out) *newB_out = c.B;
    API_CATCH
}

gsap_status gsap_apply_moves(gsap_ctx *ctx, int32_t first, int32_t count, const int32_t *s, const uint8_t *acc) {
    API_TRY
    REQUIRE(ctx && s && acc, GSAP_EINVAL, "NULL argument");
    Ctx &c = ctx->c;
    REQUIRE(first >= 0 && count >= 0 && (long long)first + count <= c.V, GSAP_EINVAL, "range out of bounds");
    // s and acc may each be host or device: both staged to the device, then
    // range-checked there before anything is written into b
    const int *ds = stage_in(c, s, (size_t)count, c.s);
    const unsigned char *da = stage_in(c, (const unsigned char *)acc, (size_t)count, c.acc);
    REQUIRE(device_ids_ok(c, count, ds, da, c.B, false), GSAP_EINVAL, "accepted s out of [0, B)");
    launch_apply(c, first, count, ds, da, nullptr, c.scal, nullptr);
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    API_CATCH
}

gsap_status gsap_move_batch(gsap_ctx *ctx, uint32_t outer, uint32_t itr, int32_t first, int32_t count,
                            int32_t *s_out, double *dS_out, uint8_t *acc_out, double *dsum_out) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    Ctx &c = ctx->c;
    REQUIRE(first >= 0 && count >= 0 && (long long)first + count <= c.V, GSAP_EINVAL, "range out of bounds");
    GSAP_CUDA(cudaMemsetAsync(c.scal, 0, sizeof(double), c.stream));
    move_batch(c, outer, itr, first, count, c.scal);
    copy_out(c, s_out, c.s, sizeof(int) * (size_t)count);
    copy_out(c, dS_out, c.dS, sizeof(double) * (size_t)count);
    copy_out(c, acc_out, c.acc, (size_t)count);
    if (dsum_out) {
        GSAP_CUDA(cudaMemcpyAsync(c.h_scal, c.scal, sizeof(double), cudaMemcpyDeviceToHost, c.stream));
        GSAP_CUDA(cudaStreamSynchronize(c.stream));
        *dsum_out = c.h_scal[0];
    }
    API_CATCH
}

gsap_status gsap_mcmc_phase(gsap_ctx *ctx, uint32_t outer, double thresh, double *D_out, int32_t *itrs_out) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    Ctx &c = ctx->c;
    REQUIRE(thresh >= 0.0, GSAP_EINVAL, "thresh must be >= 0");
    std::vector<double> D;
    const int ran = mcmc_phase(c, outer, thresh, &D);
    c.st.mcmc_itr_total += ran;
    if (D_out && ran) memcpy(D_out, D.data(), sizeof(double) * (size_t)ran);
    if (itrs_out) *itrs_out = ran;
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    API_CATCH
}

gsap_status gsap_merge_phase(gsap_ctx *ctx, uint32_t outer, int32_t K, int32_t *best_out, double *dSbest_out) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    merge_phase(ctx->c, outer, K, best_out, dSbest_out);
    GSAP_CUDA(cudaStreamSynchronize(ctx->c.stream));
    API_CATCH
}

gsap_status gsap_mdl(gsap_ctx *ctx, double *mdl_out, double *data_term_out) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    Ctx &c = ctx->c;
    const double S = device_data_term(c);
    if (data_term_out) *data_term_out = S;
    if (mdl_out) *mdl_out = model_term(c.W, c.V, c.B, c.prm.model_term) + S;
    API_CATCH
}

// export of a padded CSR / CSC (multi-kernel sparse rebuild): compacted on the host
static gsap_status get_blockmodel_padded(Ctx &c, int64_t *nnz_io, int64_t *rowptr, int32_t *col, int32_t *cnt,
                                         int32_t *cum, int64_t *colptr, int32_t *row, int32_t *ccnt, int32_t *ccum,
                                         int32_t *dout, int32_t *din) {
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    const size_t B = (size_t)c.B, E = (size_t)c.E;
    const std::vector<int> rp = to_host(c.bm_rowptr, B), re = to_host(c.bm_rowend, B);
    const std::vector<int> cp = to_host(c.bm_colptr, B), ce = to_host(c.bm_colend, B);
    int64_t nnz = 0, nnzc = 0;
    for (size_t x = 0; x < B; ++x) {
        nnz += re[x] - rp[x];
        nnzc += ce[x] - cp[x];
    }
    REQUIRE(nnz == nnzc, GSAP_ECUDA, "row / column entry counts differ");
    const bool any = col || cnt || cum || row || ccnt || ccum;
    REQUIRE(!any || *nnz_io >= nnz, GSAP_EINVAL, "entry arrays too small (see *nnz_io)");
    *nnz_io = nnz;
    auto ptr_out = [&](int64_t *dst, const std::vector<int> &p, const std::vector<int> &e) {
        if (!dst) return;
        std::vector<int64_t> w(B + 1, 0);
        for (size_t x = 0; x < B; ++x) w[x + 1] = w[x] + (e[x] - p[x]);
        GSAP_CUDA(cudaMemcpy(dst, w.data(), sizeof(int64_t) * (B + 1), cudaMemcpyDefault));
    };
    // the entries are compacted on the device (one warp per line) into dst if
    // it is device memory, else into scratch followed by one nnz-sized copy
    int *off_r = c.wa, *off_c = c.wb, *stage = reinterpret_cast<int *>(c.keys1);
    {
        std::vector<int> orow(B), ocol(B);
        int a = 0, b2 = 0;
        for (size_t x = 0; x < B; ++x) {
            orow[x] = a;
            ocol[x] = b2;
            a += re[x] - rp[x];
            b2 += ce[x] - cp[x];
        }
        if (B) {
            GSAP_CUDA(cudaMemcpy(off_r, orow.data(), sizeof(int) * B, cudaMemcpyHostToDevice));
            GSAP_CUDA(cudaMemcpy(off_c, ocol.data(), sizeof(int) * B, cudaMemcpyHostToDevice));
        }
    }
    (void)E;
    auto ent_out = [&](int32_t *dst, const int *src, bool rows) {
        if (!dst || nnz == 0) return;
        const bool dev = is_dev(dst);
        export_lines(c, rows ? c.bm_rowptr : c.bm_colptr, rows ? c.bm_rowend : c.bm_colend, rows ? off_r : off_c,
                     src, dev ? dst : stage);
        if (!dev) GSAP_CUDA(cudaMemcpyAsync(dst, stage, sizeof(int) * (size_t)nnz, cudaMemcpyDeviceToHost, c.stream));
        GSAP_CUDA(cudaStreamSynchronize(c.stream));
    };
    ptr_out(rowptr, rp, re);
    ptr_out(colptr, cp, ce);
    ent_out(col, c.bm_col, true);
    ent_out(cnt, c.bm_cnt, true);
    ent_out(cum, c.bm_cum, true);
    ent_out(row, c.bm_row, false);
    ent_out(ccnt, c.bm_ccnt, false);
    ent_out(ccum, c.bm_ccum, false);
    if (dout) GSAP_CUDA(cudaMemcpy(dout, c.dout, sizeof(int) * B, cudaMemcpyDefault));
    if (din) GSAP_CUDA(cudaMemcpy(din, c.din, sizeof(int) * B, cudaMemcpyDefault));
    return GSAP_OK;
}

gsap_status gsap_get_blockmodel(gsap_ctx *ctx, int64_t *nnz_io, int64_t *rowptr, int32_t *col, int32_t *cnt,
                                int32_t *cum, int64_t *colptr, int32_t *row, int32_t *ccnt, int32_t *ccum,
                                int32_t *dout, int32_t *din) {
    API_TRY
    REQUIRE(ctx && nnz_io, GSAP_EINVAL, "NULL argument");
    Ctx &c = ctx->c;
    if (c.padded) return get_blockmodel_padded(c, nnz_io, rowptr, col, cnt, cum, colptr, row, ccnt, ccum, dout, din);
    GSAP_CUDA(cudaMemcpyAsync(c.h_int, c.d_nnz, sizeof(int), cudaMemcpyDeviceToHost, c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    const int64_t nnz = c.h_int[0];
    const bool any = col || cnt || cum || row || ccnt || ccum;
    REQUIRE(!any || *nnz_io >= nnz, GSAP_EINVAL, "entry arrays too small (see *nnz_io)");
    *nnz_io = nnz;
    const size_t B = (size_t)c.B;
    auto widen = [&](int64_t *dst, const int *src) {
        if (!dst) return;
        std::vector<int> h = to_host(src, B + 1);
        std::vector<int64_t> w(h.begin(), h.end());
        GSAP_CUDA(cudaMemcpy(dst, w.data(), sizeof(int64_t) * (B + 1), cudaMemcpyDefault));
    };
    widen(rowptr, c.bm_rowptr);
    widen(colptr, c.bm_colptr);
    const size_t nb = sizeof(int) * (size_t)nnz;
    copy_out(c, col, c.bm_col, nb);
    copy_out(c, cnt, c.bm_cnt, nb);
    copy_out(c, cum, c.bm_cum, nb);
    copy_out(c, row, c.bm_row, nb);
    copy_out(c, ccnt, c.bm_ccnt, nb);
    copy_out(c, ccum, c.bm_ccum, nb);
    copy_out(c, dout, c.dout, sizeof(int) * B);
    copy_out(c, din, c.din, sizeof(int) * B);
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    API_CATCH
}

gsap_status gsap_get_stats(gsap_ctx *ctx, gsap_stats *out) {
    API_TRY
    REQUIRE(ctx && out, GSAP_EINVAL, "NULL argument");
    fill_stats(ctx->c, out);
    API_CATCH
}

gsap_status gsap_reset_stats(gsap_ctx *ctx) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    Ctx &c = ctx->c;
    for (KClass *k : {&c.k_move, &c.k_rebuild, &c.k_merge, &c.k_mdl, &c.k_comm, &c.k_groups, &c.k_warps}) {
        kc_resolve(c, *k);
        k->ms = 0;
        k->bytes = 0;
        k->launches = 0;
    }
    GSAP_CUDA(cudaMemsetAsync(c.n_eval, 0, sizeof(unsigned long long), c.stream));
    GSAP_CUDA(cudaStreamSynchronize(c.stream));
    c.st = gsap_stats{};
    c.launches = 0;
    API_CATCH
}

gsap_status gsap_sync(gsap_ctx *ctx) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    GSAP_CUDA(cudaStreamSynchronize(ctx->c.stream));
    API_CATCH
}

gsap_status gsap_run(gsap_ctx *ctx, int32_t *bmap_out, int32_t *B_out, double *mdl_out, double *trace,
                     int32_t trace_cap, int32_t *rounds_out) {
    API_TRY
    REQUIRE(ctx, GSAP_EINVAL, "NULL ctx");
    run_impl(ctx->c, bmap_out, B_out, mdl_out, trace, trace_cap, rounds_out);
    API_CATCH
}

gsap_status gsap_nccl_unique_id(uint8_t *id_out) {
    API_TRY
    REQUIRE(id_out, GSAP_EINVAL, "NULL argument");
    comm_unique_id(id_out);
    API_CATCH
}

gsap_status gsap_shard_slice(int32_t n, int32_t chunk, int32_t nranks, int32_t rank, int32_t *first,
                             int32_t *count, int32_t *per_rank) {
    API_TRY
    REQUIRE(n >= 0 && chunk >= 1 && nranks >= 1 && rank >= 0 && rank < nranks && first && count && per_rank,
            GSAP_EINVAL, "bad argument");
    shard_slice(n, chunk, nranks, rank, first, count, per_rank);
    API_CATCH
}

gsap_status gsap_shard_plan(gsap_ctx *ctx, int32_t first, int32_t count, int32_t nranks, int32_t *first_out,
                            int32_t *count_out) {
    API_TRY
    REQUIRE(ctx && first_out && count_out && nranks >= 1, GSAP_EINVAL, "bad argument");
    Ctx &c = ctx->c;
    REQUIRE(first >= 0 && count >= 0 && (long long)first + count <= c.V, GSAP_EINVAL, "range out of bounds");
    std::vector<int> f, n;
    shard_plan(c, first, count, nranks, f, n);
    for (int g = 0; g < nranks; ++g) {
        first_out[g] = first + f[g];
        count_out[g] = n[g];
    }
    API_CATCH
}

gsap_status gsap_partition(int32_t V, const int64_t *rowptr, const int32_t *col, const int32_t *wgt,
                           const gsap_params *params, const gsap_dist *dist, int32_t *bmap_out, int32_t *B_out,
                           double *mdl_out, gsap_stats *stats) {
    gsap_ctx *ctx = nullptr;
    const auto t0 = std::chrono::steady_clock::now();
    gsap_status st = gsap_create(V, rowptr, col, wgt, params, dist, nullptr, &ctx);
    if (st != GSAP_OK) return st;
    const double t_setup = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    st = gsap_run(ctx, bmap_out, B_out, mdl_out, nullptr, 0, nullptr);
    if (st == GSAP_OK && stats) {
        st = gsap_get_stats(ctx, stats);
        stats->t_setup = t_setup;
        stats->t_total = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    }
    const auto td = std::chrono::steady_clock::now();
    gsap_destroy(ctx);
    if (getenv("GSAP_TIMING"))
        fprintf(stderr, "[gsap] partition: create %.3f ms, destroy %.3f ms\n", 1e3 * t_setup,
                std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - td).count());
    return st;
}

}  // extern "C"
