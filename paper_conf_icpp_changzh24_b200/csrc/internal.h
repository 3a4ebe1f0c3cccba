// internal.h -- the device state owned by a gsap_ctx and the host-side entry
// points of each kernel family (rebuild.cu, move.cu, merge.cu, mdl.cu).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <functional>
#include <string>
#include <vector>

#include "../../include/gsap.h"
#include "common.cuh"

namespace gsap {

struct KClass;
// an event pair recorded inside a captured CUDA graph (re-read after every launch)
struct GraphEv {
    KClass *k;
    cudaEvent_t e0, e1;
    double bytes;
};

// timing / accounting of one kernel class (CUDA events on the context stream)
struct KClass {
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> pending;
    std::vector<cudaEvent_t> pool;
    double ms = 0.0, bytes = 0.0;
    long long launches = 0;
};

struct Ctx {
    int dev = 0;
    void *arena = nullptr;         // the single device allocation all buffers live in
    size_t arena_bytes = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    cudaStream_t side = nullptr;                 // second stream (group roles of k_move run beside the warp role)
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    gsap_params prm{};

    // graph (device): out CSR in the caller's order, in CSC (by source id, then
    // CSR position), the source of every edge, weighted degrees, self-loops
    int V = 0, E = 0;
    long long W = 0;
    bool weighted = false;
    int *rowptr = nullptr, *col = nullptr, *wgt = nullptr;
    int *cscptr = nullptr, *cscsrc = nullptr, *cscwgt = nullptr;
    int *esrc = nullptr, *kout = nullptr, *kin = nullptr, *selfw = nullptr;
    std::vector<int> h_rowptr, h_cscptr;   // host copies (static) for batch accounting
    // vertices whose total degree exceeds the warp path's table (static list)
    int *mid = nullptr, *big = nullptr, *huge = nullptr;   // 128 < k <= 256 / <= 1024 / > 1024 entries
    int *midbig = nullptr;                                 // 128 < k <= 1024 (latency mode's CTA list)
    std::vector<int> h_mid, h_big, h_huge, h_midbig;
    size_t big_table_slots = 0;            // per-CTA global table capacity (slots)
    int *big_tables = nullptr;             // global tables for very large vertices

    // partition
    int *b = nullptr;
    int B = 0;
    // neighbour-block cache: nbo[p] = b[col[p]] for every out-CSR
    // position p, nbi[q] = b[cscsrc[q]] for every in-CSC position q, so the
    // kernels that need the blocks of a vertex's neighbours read them with the
    // adjacency (coalesced) instead of gathering b per entry.  Kept up to date
    // by the apply of every MOVE batch (k_nb_update: only the moved vertices'
    // entries, through the CSC <-> CSR position maps); any other change of b
    // (create, set_partition, merges, bracket restores) marks it stale and the
    // next rebuild refreshes it in full (k_nb_refresh).
    int *nbo = nullptr, *nbi = nullptr, *csc2csr = nullptr, *csr2csc = nullptr;
    bool nb_stale = true;
    // the update after a MOVE batch runs on the side stream beside the dense-regime
    // rebuild (which does not read the cache); every reader or writer of nbo / nbi
    // joins it first (nb_join)
    bool nb_pending = false;
    // sparse regime with the persistent rebuild: the update after an apply is
    // deferred into that rebuild's first phase (nb_flush launches it on its own
    // if anything else needs the cache first)
    bool nb_deferred = false;
    cudaEvent_t ev_nb = nullptr, ev_apply = nullptr;

    // blockmodel (capacity: nnz <= min(E, B^2); B <= V)
    int *bm_rowptr = nullptr, *bm_col = nullptr, *bm_cnt = nullptr, *bm_cum = nullptr;
    int *bm_colptr = nullptr, *bm_row = nullptr, *bm_ccnt = nullptr, *bm_ccum = nullptr;
    int *dout = nullptr, *din = nullptr, *d_nnz = nullptr;
    // padded CSR/CSC (multi-kernel sparse rebuild): line x = [ptr[x], end[x]) inside
    // its counting-sort segment [ptr[x], ptr[x + 1]), cnt = 0 in the padding and
    // d_nnz = E (the extent the MDL sums over); otherwise compact (end = ptr + 1)
    bool padded = false;
    int *bm_rowend = nullptr, *bm_colend = nullptr;
    int *dense = nullptr, *denseT = nullptr;
    double2 *ft = nullptr;         // f-table {hi, lo} (FT_N entries)
    double *rcp = nullptr;         // 1 / (d_x + B), refreshed by every rebuild
    int *mt = nullptr;             // N4: the shared multinomial table (one neighbour block per block)
    size_t dense_cap = 0;   // elements
    bool dense_mode = false;
    int dense_B = -1;       // B of the dense M / Mt the last rebuild left (-1: none)

    // rebuild scratch
    unsigned long long *keys0 = nullptr, *keys1 = nullptr, *vals64a = nullptr, *vals64b = nullptr;
    unsigned *ukeys0 = nullptr, *ukeys1 = nullptr;
    int *wa = nullptr, *wb = nullptr, *flags = nullptr, *pos = nullptr, *tmpi = nullptr,
        *counts = nullptr, *scan_tmp = nullptr, *rownnz = nullptr;
    size_t counts_cap = 0, scan_tmp_cap = 0;
    // segmented rebuild scratch (per line: length, offset, cursor, runs; line lists)
    int *seg_len = nullptr, *seg_cur = nullptr, *seg_nnz = nullptr, *seg_listW = nullptr,
        *seg_listC = nullptr, *seg_ctr = nullptr, *xl_hp = nullptr, *seg_listM = nullptr;
    unsigned long long *xl_keys = nullptr;   // 2E: long-segment sort scratch
    // persistent sparse rebuild (coop.cuh; small graphs): the column side's
    // line scratch, its long-segment scratch, the grid barrier
    bool coop_ok = false;
    int *seg2_len = nullptr, *seg2_cur = nullptr, *seg2_nnz = nullptr, *seg2_listC = nullptr;
    // the multi-kernel rebuild's column side (runs beside the rows on the side stream)
    int *seg2_listW = nullptr, *seg2_listM = nullptr, *seg2_ctr = nullptr, *scan_tmp2 = nullptr;
    cudaEvent_t ev_rb_fork = nullptr, ev_rb_join = nullptr;
    unsigned long long *xl2_keys = nullptr;
    int *xl2_hp = nullptr;
    unsigned *coop_bar = nullptr;
    // persistent dense rebuild for B <= SMALL_MAX_B (params.dense_coop): B^2 accumulator, zero between calls
    int *small_acc = nullptr;

    // per-phase buffers
    int *s = nullptr;            // proposals: V (MOVE) or B * P (MERGE)
    double *dS = nullptr;        // V or B * P
    double *H = nullptr;         // V
    unsigned char *acc = nullptr;// V
    int *best = nullptr;         // B
    double *dSbest = nullptr;    // B
    double *partials = nullptr;  // reduction partials
    double *bpart = nullptr;     // MCMC graphs: the accepted-dS chunk partials of every batch of an iteration
    double *scal = nullptr;      // device scalars [0] = batch dS sum, [1] = data term
    int *scal_i = nullptr;       // device int scalars [0] = new B, [1] = accepted moves, [4] apply
                                 // arrivals, [6] argument check flag
    unsigned long long *n_eval = nullptr;   // device counter: evaluated MOVE proposals (s != b[v])
    double *Dh = nullptr;        // per-iteration sum of accepted dS (max_nodal_itr)
    // sorted two-pass MOVE (move.cu): per-block counts / offsets [2B], the batch
    // grouped by r then by s [2 count], pass-1 partials [3 count], scan scratch
    int *mv_cnt = nullptr, *mv_perm = nullptr, *mv_scan_tmp = nullptr;
    double *mv_part = nullptr;
    int *slot_b[3] = {nullptr, nullptr, nullptr};   // golden-section bracket partitions
    // merge selection scratch
    unsigned long long *skey0 = nullptr, *skey1 = nullptr;
    int *sval0 = nullptr, *sval1 = nullptr, *sel_rank = nullptr, *nxt0 = nullptr, *nxt1 = nullptr,
        *mx0 = nullptr, *mx1 = nullptr, *oncyc = nullptr, *label = nullptr, *present = nullptr;

    // pinned host scalars
    double *h_scal = nullptr;
    int *h_int = nullptr;

    // multi-GPU (nranks > 1), or one process emulating prm.sim_ranks ranks
    int nranks = 1, rank = 0;
    void *nccl_comm = nullptr;
    int batch_count = 0;           // the MOVE batch a launch belongs to (mode decisions per batch, not slice)
    int test_grid = 0;             // tests (env GSAP_TEST_GRID at create): cap of the move kernels' grids

    // N2 incremental update (dense regime): the batch a pending rebuild follows;
    // the apply logs moved vertices and their old blocks, the rebuild applies dM
    struct DeltaBatch {
        int first = 0, count = 0;
        const unsigned char *acc = nullptr;
        bool pending = false;
    } delta;
    int *oldb = nullptr, *moved = nullptr, *moved_cnt = nullptr;
    int *movedb = nullptr;                      // the new block of each logged move (k_nb_update)
    int *dnnz_r = nullptr, *dnnz_c = nullptr;   // dense regime: non-zeros per row of M / of Mt (kept for N2)
    // dense regime above SMALL_MAX_B: the lines of M padded to B entries (line
    // x at x B); N2 marks the lines a batch changed and re-compacts only those
    bool dense_padded = false;
    unsigned char *line_dirty = nullptr;   // [2 B]: rows of M, then rows of Mt
    unsigned *dl_arrive = nullptr;         // last-CTA counter of k_dense_lines

    // CUDA-graph capture of an MCMC iteration (N1: launch overhead, §5)
    unsigned *d_itr = nullptr;     // MCMC iteration read by k_move (device scalar)
    // the instantiated graph of the last MCMC phase, updated in place
    // (cudaGraphExecUpdate) by the next phase's capture when the topology is
    // the same -- one instantiation per regime instead of one per round
    cudaGraphExec_t mcmc_exec = nullptr;
    int mcmc_exec_mode = 0;        // 1: one graph per iteration, 2: the device-side loop
    bool capturing = false;
    std::vector<GraphEv> graph_ev;

    // accounting
    long long launches = 0;
    KClass k_move, k_rebuild, k_merge, k_mdl, k_comm;
    KClass k_groups, k_warps;   // profile mode, outside graphs: the two MOVE roles timed on their own streams
    gsap_stats st{};
    std::vector<double> move_bytes_per_batch;   // algorithmic bytes per MOVE launch

    BM bm() const {
        BM m;
        m.B = B;
        m.dense = dense_mode ? dense : nullptr;
        m.ft = ft;
        m.rcp = rcp;
        m.rowptr = bm_rowptr; m.col = bm_col; m.cnt = bm_cnt; m.cum = bm_cum;
        m.colptr = bm_colptr; m.row = bm_row; m.ccnt = bm_ccnt; m.ccum = bm_ccum;
        m.rowend = padded ? bm_rowend : bm_rowptr + 1;
        m.colend = padded ? bm_colend : bm_colptr + 1;
        m.dout = dout; m.din = din;
        m.mt = prm.proposal_mode == 1 ? mt : nullptr;
        return m;
    }
};

// error plumbing -----------------------------------------------------------
struct Error {
    gsap_status code;
    std::string msg;
};

#define GSAP_CUDA(x)                                                                          \
    do {                                                                                      \
        cudaError_t e_ = (x);                                                                 \
        if (e_ != cudaSuccess)                                                                \
            throw ::gsap::Error{GSAP_ECUDA, std::string(#x) + ": " + cudaGetErrorString(e_)}; \
    } while (0)

#define GSAP_CHECK_LAUNCH() GSAP_CUDA(cudaGetLastError())

// f() once per (key, current device), result cached under a mutex: kernel
// attributes (cudaFuncSetAttribute is per device) and occupancy-derived grids
int per_device(const void *key, const std::function<int()> &f);

// event timing of a kernel class (no-op unless prm.profile)
void kc_begin(Ctx &c, KClass &k, cudaEvent_t *ev);
void kc_end(Ctx &c, KClass &k, cudaEvent_t ev, double bytes);
void kc_resolve(Ctx &c, KClass &k);
cudaEvent_t role_begin(Ctx &c, KClass &k, cudaStream_t st);
void role_end(Ctx &c, KClass &k, cudaEvent_t e0, cudaStream_t st);

// rebuild.cu
void build_graph_device(Ctx &c);                 // CSC, esrc, degrees (create time)
void nb_refresh(Ctx &c);                         // the neighbour-block cache from b (if stale)
inline void b_changed(Ctx &c) { c.nb_stale = true; }   // every bulk write of b outside the apply
void nb_join(Ctx &c, bool flush = true);         // the main stream waits for a pending cache update
void nb_flush(Ctx &c);                           // a deferred cache update launched now (then joined)
void rebuild(Ctx &c);                            // Alg. 2 from c.b, c.B
bool dense_ok(const Ctx &c, int B);
// padded-CSR export: line x's [ptr[x], end[x]) of src to dst[off[x] ..) on the device
void export_lines(Ctx &c, const int *ptr, const int *end, const int *off, const int *src, int *dst);
constexpr int SMALL_MAX_B = 221;               // B^2 ints in one CTA's shared memory (195 KB)

// move.cu
enum MoveMode { MOVE_FUSED = 0, MOVE_PROPOSE = 1, MOVE_DELTA = 2 };
void launch_move(Ctx &c, MoveMode mode, uint32_t outer, uint32_t itr, int first, int count,
                 int *s, double *dS, double *H, unsigned char *acc, const unsigned *d_itr = nullptr);
void launch_apply(Ctx &c, int first, int count, const int *s, const unsigned char *acc,
                  const double *dS, double *dsum, int *nacc, unsigned long long *n_eval = nullptr);
// device-side range check of id arrays (argument validation); synchronises
bool device_ids_ok(Ctx &c, int n, const int *x, const unsigned char *mask, int B, bool not_self);

void launch_partials(Ctx &c, int first, int count, const int *s, const unsigned char *acc, const double *dS,
                     double *partials);
// the apply of a batch inside an MCMC graph: b, counters, move log and cache
// update as launch_apply, the chunk partials into part[] only -- the
// iteration's ordered sum is taken once by launch_data_term(c, &dsum_spec)
void launch_apply_deferred(Ctx &c, int first, int count, const int *s, const unsigned char *acc, const double *dS,
                           double *part, int *nacc, unsigned long long *n_eval);
void launch_apply_gathered(Ctx &c, int first, int count, const int *s, const unsigned char *acc,
                           const double *partials, int n, double *dsum, int *nacc,
                           unsigned long long *n_eval = nullptr);
constexpr int APPLY_CHUNK_V = 1024;   // fixed reduction chunk of the accepted-dS sums (move.cu)

// comm.cu: multi-GPU (one process per GPU, NCCL over NVLink, loaded at run time)
void comm_init(Ctx &c, const gsap_dist *d);
void comm_destroy(Ctx &c);
void comm_allgather(Ctx &c, void *recv, size_t count_per_rank, int dtype);   // dtype: 0 int8, 1 int32, 2 f64
// in place, variable slices (rank g: cnt[g] elements at off[g]); contiguous result
void comm_allgatherv(Ctx &c, void *buf, const std::vector<int> &off, const std::vector<int> &cnt, int dtype);
// a MOVE batch cut into G edge-balanced slices of whole APPLY_CHUNK_V chunks (offsets relative to first)
void shard_plan(const Ctx &c, int first, int count, int G, std::vector<int> &off, std::vector<int> &cnt);
void comm_unique_id(uint8_t out[128]);
// the slice of [0, n) that rank g of G owns: whole chunks of `chunk`, contiguous,
// ceil(ceil(n/chunk)/G) chunks per rank (the last ranks may own less or none)
void shard_slice(int n, int chunk, int G, int g, int *first, int *count, int *per_rank);

// N4 ablation: fill the shared neighbour-block table for a merge phase
// (phase 0, j = TABLE_J) or a MOVE batch (phase 1, j = TABLE_J | first)
void launch_fill_mt(Ctx &c, uint32_t j, uint32_t itr, uint32_t outer, uint32_t phase,
                    const unsigned *d_itr = nullptr);

// merge.cu
void launch_merge_props(Ctx &c, uint32_t outer, int first, int count, bool propose, int *s,
                        double *dS, int *best, double *dSbest);
void select_merges(Ctx &c, const int *best, const double *dS, int K, int *label_out);

// mdl.cu
// the iteration's sum of accepted dS from the batches' chunk partials (batch k
// at part + k stride: nch_first chunks, the last batch nch_last), in the order
// of k_apply_sum's running sum -> c.scal[0]
struct DsumSpec {
    const double *part;
    int nbat, stride, nch_first, nch_last;
};
void launch_data_term(Ctx &c, const DsumSpec *dsum = nullptr);   // -> c.scal[1] (and [0]), no synchronisation
double device_data_term(Ctx &c);                 // S = -sum f(M) + sum f(dout) + sum f(din)
double model_term(long long W, int V, int B, int variant);

}  // namespace gsap
