/*
 * gsap.h -- C-ABI of the B200 (sm_100a) implementation of the hot path of
 * GSAP's stochastic block partitioning (Chang, Zhang & Huang, ICPP'24).
 *
 * Citations "P:<line> <section>" refer to the paper text; "R:Zn"
 * to the readings of the paper listed in DESIGN.md.  Problem statement:
 * a directed graph G in CSR (optional integer edge weights) in; a partition
 * Bmap (vertex -> block) and the block count B* minimising the description
 * length of Eq. 2 out (P:52-63 2.1, Alg. 2).
 *
 * Conventions (all entry points):
 *   - Every function returns gsap_status; nothing throws or aborts across the
 *     ABI.  gsap_last_error() gives a thread-local message for the last error.
 *   - Ownership: the caller owns every buffer it passes.  gsap_create copies the
 *     graph; the context owns all device state and frees it in gsap_destroy.
 *   - Pointer arguments marked "host or device" may point to host memory or
 *     to device memory of the context's GPU (told apart with
 *     cudaPointerGetAttributes, each pointer separately).  Outputs, host or
 *     device, are complete when the call returns (the call synchronises the
 *     context's stream), so a device output may be read on any stream.
 *     Device INPUTS are read on the context's stream: the caller must have
 *     completed the work that produced them (e.g. synchronised its stream)
 *     before the call.  Device id inputs are range-checked on the device
 *     before any state changes (GSAP_EINVAL otherwise).
 *   - Ids are 0-based.  Vertex ids are int32, edge offsets int64 at the ABI.
 *   - Limits: 1 <= V < 2^31, number of edges and total edge weight < 2^30,
 *     weights >= 1 (GSAP_EUNSUPPORTED / GSAP_EINVAL otherwise).
 *   - After GSAP_ECUDA or GSAP_ENCCL the context must be destroyed; any other
 *     error leaves it valid and unchanged.
 *   - The library runs only on sm_100 devices; there is no CPU fallback.
 */
#ifndef GSAP_H
#define GSAP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    GSAP_OK = 0,
    GSAP_EINVAL = 1,        /* bad argument (range, NULL, malformed CSR) */
    GSAP_ENOMEM = 2,        /* device or host allocation failed */
    GSAP_ECUDA = 3,         /* CUDA runtime error (context must be destroyed) */
    GSAP_ENCCL = 4,         /* NCCL error (context must be destroyed) */
    GSAP_ESTATE = 5,        /* call order (e.g. a phase needs B >= 2) */
    GSAP_EUNSUPPORTED = 6   /* size limits, or not an sm_100 device */
} gsap_status;

typedef enum { GSAP_MERGE = 0, GSAP_MOVE = 1 } gsap_phase;

/* SBP parameters: Table 2 (P:295-305 4.1) + readings Z3-Z5, Z10 */
#define GSAP_COOP_MAX_E (1 << 23)

typedef struct {
    uint64_t seed;            /* Philox key (R:O.3); default 0x5B9D2024 */
    double beta;              /* MH inverse temperature (R:Z5); default 3 */
    double reduction_rate;    /* num_blocks_reduction_rate; default 0.4 */
    int32_t num_proposals;    /* merge proposals per block; default 10 */
    int32_t max_nodal_itr;    /* max MCMC iterations per round; default 100 */
    double thresh1;           /* delta_entropy_threshold1; default 5e-4 */
    double thresh2;           /* delta_entropy_threshold2; default 1e-4 */
    int32_t window;           /* delta_entropy_moving_avg_window; default 3 */
    int32_t num_batches;      /* num_batches_for_MCMC; default 4 */
    int32_t model_term;       /* 0: E h(B^2/E) (Eq. 2); 1: GraphChallenge variant (R:Z3) */
    int32_t max_rounds;       /* guard on merge+MCMC rounds; default 500 */
    int32_t profile;          /* 1: time kernels with CUDA events (gsap_stats k_*) */
    int32_t cuda_graphs;      /* 0: plain launches; 1: each MCMC iteration one CUDA graph launch;
                                 2 (default): the whole MCMC phase one graph launch, a device-side
                                 while loop (conditional node) with the convergence test on the GPU
                                 (profile = 1 or multi-GPU runs use 1).  Either way the executable
                                 graph is kept and updated in place by the next round's capture. */
    int32_t dense_max_B;      /* dense blockmodel iff B <= this; 0 = auto (B^2 <= max(8E, 2^24)) */
    int32_t sparse_coop;      /* 1 (default): sparse-regime rebuild as one persistent kernel when
                                 E <= GSAP_COOP_MAX_E; 0: the multi-kernel rebuild (same result) */
    int32_t dense_coop;       /* dense-regime rebuild: 1 (default) one persistent kernel when
                                 B <= 221 (shared-memory histogram), the multi-kernel path above;
                                 2: the persistent kernel for every dense B (L2 atomics above 221;
                                 slower there on B200); 0: always multi-kernel.  Same result. */
    int32_t sel_small;        /* 1 (default): merge selection (a4) for B <= 4096 in one CTA (shared
                                 memory) + 4 grid launches; 0: the multi-kernel selection (radix
                                 sort, pointer-doubling launches).  Same result. */
    int32_t move_sorted;      /* MOVE batches in the sparse regime: 1 (default) the sorted two-pass
                                 evaluation (batch grouped by r, then by s) for graphs of
                                 more than GSAP_COOP_MAX_E edges and batches of >= 2^16 vertices;
                                 2: always (sparse regime, B > 128); 0: never (one fused pass).
                                 Same integers; dS sums in another order (1e-9 contract). */
    int32_t sim_ranks;        /* verification mode (tests): > 1 runs the multi-GPU data path of
                                 sim_ranks ranks in ONE process on one GPU -- every MOVE batch and
                                 merge phase cut into the ranks' slices exactly as with NCCL, each
                                 slice computed in rank order, the all-gathers skipped (the slices
                                 already sit at their offsets); default 0 = off */
    int32_t incremental;      /* N2 (P:250-255 3.4): 1 (default) the rebuild after a MOVE batch in the
                                 dense regime applies the change of M by the batch's moves to the
                                 previous M (and skips the compaction when nothing moved); 0: every
                                 rebuild from scratch.  Same blockmodel bit for bit. */
    int32_t proposal_mode;    /* 0 (default): a fresh Philox draw per proposal (R:Z6).  1: the paper-
                                 literal lookup-table ablation (N4; Alg. 1, Fig. 4):
                                 ONE weighted neighbour block per block, drawn per merge phase / MOVE
                                 batch and shared by every proposal that reaches that block (a MERGE
                                 outcome equal to r is redrawn uniformly over the other blocks) */
    int32_t line_sort;        /* multi-kernel sparse rebuild of an unweighted graph: 1 (default) lines of
                                 129..1024 entries sorted by one bucket pass + insertion sorts inside the
                                 buckets (k_segsort_bucket); 0: register bitonic / warp radix sorts.
                                 Same blockmodel bit for bit. */
} gsap_params;

/* multi-GPU: one process per GPU; NULL or nranks == 1 means single GPU (see gsap_nccl_unique_id) */
typedef struct {
    int32_t nranks, rank, device;
    uint8_t nccl_id[128];     /* ncclUniqueId from rank 0, broadcast by the caller */
} gsap_dist;

typedef struct {
    double t_total, t_setup, t_merge, t_move, t_mdl;   /* host wall seconds */
    int64_t n_move_prop, n_move_acc, n_merge_prop;      /* proposals generated / accepted */
    int32_t rounds, mcmc_itr_total, B_final;
    int64_t gpu_launches;                               /* kernels launched by the library */
    /* device time (CUDA events on the context stream, profile = 1) and the
     * algorithmic HBM bytes of each kernel class */
    double k_move_ms, k_move_bytes; int64_t k_move_launches;
    double k_rebuild_ms, k_rebuild_bytes; int64_t k_rebuild_launches;
    double k_merge_ms, k_merge_bytes; int64_t k_merge_launches;
    double k_mdl_ms; int64_t k_mdl_launches;
    /* device seconds of the blockmodel rebuilds (Alg. 2) and of
     * the multi-GPU exchange (both profile = 1, else 0), and the MOVE
     * proposals actually evaluated (s != b[v]; R:Z13 makes the rest no-ops) */
    double t_rebuild, t_comm;
    int64_t n_move_eval;
} gsap_stats;

typedef struct gsap_ctx gsap_ctx;

/* Table 2 defaults into *p. */
void gsap_default_params(gsap_params *p);

/* Thread-local message of the last non-OK status ("" if none). */
const char *gsap_last_error(void);

/*
 * One-shot SBP (P:137-141 3, Fig. 2): merge -> batched MCMC -> golden-section
 * until the MDL-optimal B.  rowptr[V+1] (int64), col[E] (int32), wgt[E]
 * (int32, NULL = all 1): host or device, read-only.  bmap_out[V]: host or
 * device; labels in [0, B_out).  B_out, mdl_out: host.  stats: host, nullable.
 * dist: nullable (single GPU).  Blocking.
 */
gsap_status gsap_partition(int32_t V, const int64_t *rowptr, const int32_t *col,
                           const int32_t *wgt, const gsap_params *params,
                           const gsap_dist *dist, int32_t *bmap_out, int32_t *B_out,
                           double *mdl_out, gsap_stats *stats);

/*
 * Stepwise interface (parity tests, benches).  gsap_create copies the graph
 * (host or device pointers) to the device, builds the in-edge CSC, sets the
 * singleton partition b = iota (B = V, P:61 2.1) and rebuilds the blockmodel.
 * stream: a cudaStream_t of the current device, or NULL (the context then
 * creates its own non-blocking stream).
 */
gsap_status gsap_create(int32_t V, const int64_t *rowptr, const int32_t *col,
                        const int32_t *wgt, const gsap_params *params,
                        const gsap_dist *dist, void *stream, gsap_ctx **out);
void gsap_destroy(gsap_ctx *ctx);

/* Replace b (host or device, V entries in [0, B)) and B; rebuilds (Alg. 2). */
gsap_status gsap_set_partition(gsap_ctx *ctx, const int32_t *b, int32_t B);
/* Copy b out (host or device, V entries); *B_out (host) = current B. */
gsap_status gsap_get_partition(gsap_ctx *ctx, int32_t *b_out, int32_t *B_out);

/* Blockmodel rebuild from the context's b (Alg. 2, P:257-283 3.4). */
gsap_status gsap_update_blockmodel(gsap_ctx *ctx);

/*
 * Proposals (Alg. 1, P:164-201 3.2; R:O.4, Z6-Z9).  MOVE: one proposal per
 * vertex v in [first, first+count), Philox counter (v, 0, itr, outer<<1|1),
 * s_out[count].  MERGE: num_proposals per block r in [first, first+count),
 * counter (r, j, 0, outer<<1|0), s_out[count*num_proposals] (row-major).
 * proposal_mode = 1 (N4): the shared table is drawn first (MOVE: keyed by
 * `first`, the batch's first vertex; MERGE: by outer).  s_out: host or device.
 */
gsap_status gsap_propose(gsap_ctx *ctx, gsap_phase phase, uint32_t outer, uint32_t itr,
                         int32_t first, int32_t count, int32_t *s_out);

/*
 * Delta MDL (Eq. 3-7, P:205-246 3.3, exact form R:Z11, Z12).  dS = S(after) -
 * S(before) in nats (negative = better).  MOVE: s[count] proposals for
 * vertices [first, first+count); also the Hastings ratio H_out[count]
 * (nullable; R:Z5, Z26) and the MH decision acc_out[count] (nullable): accept
 * iff (w3 + 1/2) 2^-32 <= exp(-beta dS) H with w3 from the vertex's Philox
 * counter.  s == b[v] gives dS = 0, H = 1, acc = 0 (R:Z13).  MERGE:
 * s[count*num_proposals], dS_out[count*num_proposals]; H_out, acc_out unused.
 * All arrays host or device.  Reads the current (snapshot) state only.
 */
gsap_status gsap_delta_mdl(gsap_ctx *ctx, gsap_phase phase, uint32_t outer, uint32_t itr,
                           int32_t first, int32_t count, const int32_t *s,
                           double *dS_out, double *H_out, uint8_t *acc_out);

/*
 * Perform-merge (P:141 3, P:232 3.3; R:Z16-Z18): blocks ordered by (dS[r], r)
 * ascending (-0.0 == +0.0); edges r -> best[r] applied in that order as the
 * sequential GraphChallenge loop would, until K merges; b relabelled to the
 * ranks of the labels present; B := #labels present; blockmodel rebuilt.
 * best[B], dS[B]: host or device.  label_out[B] (host or device, nullable):
 * new label of each old block (-1 if its group holds no vertex).
 * newB_out: host, nullable.  Requires 0 <= K <= 0.4 B-ish (K < B/2 + 1).
 */
gsap_status gsap_select_merges(gsap_ctx *ctx, const int32_t *best, const double *dS,
                               int32_t K, int32_t *label_out, int32_t *newB_out);

/* The "apply" step of a batch (P:141 3, P:176 3.2; R:Z10): b[first+i] = s[i]
 * where acc[i] != 0.  s[count] int32, acc[count] uint8, each host or device;
 * accepted s[i] must lie in [0, B) (GSAP_EINVAL, nothing written, otherwise).
 * No rebuild (call gsap_update_blockmodel). */
gsap_status gsap_apply_moves(gsap_ctx *ctx, int32_t first, int32_t count,
                             const int32_t *s, const uint8_t *acc);

/*
 * One MCMC batch, fused (the hot loop): propose + dS + Hastings
 * + accept for vertices [first, first+count) on the batch-start snapshot,
 * apply, rebuild.  Optional outputs (host or device, nullable): s_out, dS_out,
 * acc_out [count]; dsum_out (host, nullable): sum of accepted dS.
 */
gsap_status gsap_move_batch(gsap_ctx *ctx, uint32_t outer, uint32_t itr, int32_t first,
                            int32_t count, int32_t *s_out, double *dS_out, uint8_t *acc_out,
                            double *dsum_out);

/*
 * One merge phase: every block proposes
 * num_proposals merges, best per block (first j wins ties), K merges carried
 * out, relabel, rebuild.  best_out[B], dSbest_out[B] (host or device,
 * nullable) report the per-block winners before the merge.
 */
gsap_status gsap_merge_phase(gsap_ctx *ctx, uint32_t outer, int32_t K,
                             int32_t *best_out, double *dSbest_out);

/*
 * One MCMC phase (P:141 3, P:176 3.2; Table 2; R:O.8, Z10, Z19,
 * Z20) from the current state: iterations of num_batches fused batches (ids
 * in contiguous ranges of ceil(V/num_batches)) until the GraphChallenge test
 * -mean(D[itr-w+1 : itr)) < thresh * MDL (w = params.window, MDL after the
 * iteration) or max_nodal_itr stops it.  D_out (host, nullable,
 * max_nodal_itr doubles): D[itr] = sum of the accepted dS of iteration itr;
 * itrs_out (host, nullable): iterations run.  outer keys the Philox streams.
 */
gsap_status gsap_mcmc_phase(gsap_ctx *ctx, uint32_t outer, double thresh, double *D_out, int32_t *itrs_out);

/* MDL of the current state, Eq. 2 (R:Z1-Z4, Z22); data term S (nullable). Host outputs. */
gsap_status gsap_mdl(gsap_ctx *ctx, double *mdl_out, double *data_term_out);

/*
 * Blockmodel export, the "six arrays" of P:152-159 3.1 (Fig. 3) plus the
 * block degrees of P:162 (CSR rows ascending column; CSC columns ascending row;
 * cum = inclusive prefix of cnt within a row / column).  *nnz_io (host): in =
 * capacity of the entry arrays, out = nnz.  Any array may be NULL; with all
 * arrays NULL this is a size query.  rowptr/colptr[B+1] int64; col, cnt, cum,
 * row, ccnt, ccum [nnz] int32; dout, din [B] int32.  Host or device.
 */
gsap_status gsap_get_blockmodel(gsap_ctx *ctx, int64_t *nnz_io, int64_t *rowptr, int32_t *col,
                                int32_t *cnt, int32_t *cum, int64_t *colptr, int32_t *row,
                                int32_t *ccnt, int32_t *ccum, int32_t *dout, int32_t *din);

/* Statistics accumulated since create / the last reset (host): the counts
 * behind the metric of SURVEY 8(d) (proposals, evaluations, accepts) and the
 * per-phase times of Fig. 11/12 (P:322-330 4.3). */
gsap_status gsap_get_stats(gsap_ctx *ctx, gsap_stats *out);
gsap_status gsap_reset_stats(gsap_ctx *ctx);

/* Synchronise the context's stream (host-side ordering only; no computation). */
gsap_status gsap_sync(gsap_ctx *ctx);

/*
 * Full SBP on an existing context (gsap_partition without the copy-in):
 * restarts from b = iota.  bmap_out: host or device, nullable.
 * trace (host, nullable): GSAP_TRACE_COLS doubles per round, at most
 * trace_cap rows: [outer, B after merge, MCMC iterations, MDL, round seconds,
 * accepted moves, device ms of the move / rebuild / merge kernels (profile = 1,
 * else 0), convergence threshold used (R:Z19), B before the merge (the
 * bracket slot the round restarted from, O.9), merges K requested];
 * *rounds_out (host, nullable).
 */
#define GSAP_TRACE_COLS 12
gsap_status gsap_run(gsap_ctx *ctx, int32_t *bmap_out, int32_t *B_out, double *mdl_out,
                     double *trace, int32_t trace_cap, int32_t *rounds_out);

/*
 * Multi-GPU: one process per GPU, every rank passes the same
 * graph and a gsap_dist {nranks, rank, device, nccl_id}; each MOVE batch and
 * each merge phase is split into contiguous slices (MOVE: edge-balanced runs of
 * whole 1024-vertex chunks, gsap_shard_plan; MERGE: equal block ranges), whose
 * results are exchanged in place (one ncclBroadcast per rank in one group: an
 * all-gather of variable slices); every rank then applies them identically.
 * Results are bit-identical for any nranks (verified on one GPU with
 * params.sim_ranks).  Statistics: n_move_prop / n_merge_prop count the
 * proposals of this rank's slices; n_move_acc / n_move_eval the whole batch.
 * gsap_nccl_unique_id: rank 0 creates the id (host, 128 bytes) and the caller
 * broadcasts it (e.g. with torch.distributed).  NCCL is loaded at run time.
 */
gsap_status gsap_nccl_unique_id(uint8_t *id_out);

/*
 * The slice of [0, n) rank `rank` of `nranks` owns: ceil(ceil(n/chunk)/nranks)
 * whole chunks per rank, contiguous, in rank order (the last ranks may own
 * fewer or none).  Host outputs: *first, *count, *per_rank (= the padded
 * all-gather block, in elements).  Pure host function (no device needed).
 */
gsap_status gsap_shard_slice(int32_t n, int32_t chunk, int32_t nranks, int32_t rank, int32_t *first,
                             int32_t *count, int32_t *per_rank);

/*
 * The slices a MOVE batch [first, first + count) is cut into for nranks ranks
 * (SURVEY 8(e)): contiguous, whole 1024-vertex chunks from the batch start,
 * balanced by each chunk's work (adjacency entries + 16 per vertex), the last
 * rank taking the rest.  Host outputs first_out[nranks] (absolute vertex ids)
 * and count_out[nranks].  Host-only (the graph's degrees from ctx).
 */
gsap_status gsap_shard_plan(gsap_ctx *ctx, int32_t first, int32_t count, int32_t nranks, int32_t *first_out,
                            int32_t *count_out);

#ifdef __cplusplus
}
#endif

#endif /* GSAP_H */
