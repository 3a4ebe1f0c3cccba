// comm.cu -- multi-GPU plumbing: one process per GPU, the
// graph, partition and blockmodel replicated, each MOVE batch and each merge
// phase split into contiguous slices (whole fixed-size chunks) across the
// ranks, the slices' results exchanged with ncclAllGather over NVLink /
// NVSwitch, then applied identically everywhere.  Randomness is keyed by
// global ids and every floating-point sum is over fixed chunks in a fixed
// order, so the partition is bit-identical for any number of GPUs.
//
// NCCL is loaded at run time (dlopen "libnccl.so.2": the copy torch loaded,
// or the system one), so the library has no link-time NCCL dependency.
#include <dlfcn.h>
#include <nccl.h>

#include <mutex>

#include "internal.h"

namespace gsap {

struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId *);
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int);
    ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t);
    ncclResult_t (*Broadcast)(const void *, void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*GroupStart)();
    ncclResult_t (*GroupEnd)();
    ncclResult_t (*CommDestroy)(ncclComm_t);
    const char *(*GetErrorString)(ncclResult_t);
};

static NcclApi *nccl_api() {
    static NcclApi api;
    static bool ok = false;
    static std::once_flag once;
    std::call_once(once, [] {
        void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) return;
        api.GetUniqueId = (decltype(api.GetUniqueId))dlsym(h, "ncclGetUniqueId");
        api.CommInitRank = (decltype(api.CommInitRank))dlsym(h, "ncclCommInitRank");
        api.AllGather = (decltype(api.AllGather))dlsym(h, "ncclAllGather");
        api.Broadcast = (decltype(api.Broadcast))dlsym(h, "ncclBroadcast");
        api.GroupStart = (decltype(api.GroupStart))dlsym(h, "ncclGroupStart");
        api.GroupEnd = (decltype(api.GroupEnd))dlsym(h, "ncclGroupEnd");
        api.CommDestroy = (decltype(api.CommDestroy))dlsym(h, "ncclCommDestroy");
        api.GetErrorString = (decltype(api.GetErrorString))dlsym(h, "ncclGetErrorString");
        ok = api.GetUniqueId && api.CommInitRank && api.AllGather && api.Broadcast && api.GroupStart &&
             api.GroupEnd && api.CommDestroy && api.GetErrorString;
    });
    if (!ok) throw Error{GSAP_ENCCL, "libnccl.so.2 not found (dlopen)"};
    return &api;
}

#define GSAP_NCCL(x)                                                                          \
    do {                                                                                      \
        ncclResult_t r_ = (x);                                                                \
        if (r_ != ncclSuccess)                                                                \
            throw Error{GSAP_ENCCL, std::string(#x) + ": " + nccl_api()->GetErrorString(r_)}; \
    } while (0)

void comm_unique_id(uint8_t out[128]) {
    ncclUniqueId id;
    GSAP_NCCL(nccl_api()->GetUniqueId(&id));
    memcpy(out, id.internal, 128);
}

void comm_init(Ctx &c, const gsap_dist *d) {
    c.nranks = 1;
    c.rank = 0;
    if (!d || d->nranks <= 1) return;
    if (d->rank < 0 || d->rank >= d->nranks) throw Error{GSAP_EINVAL, "dist.rank out of range"};
    ncclUniqueId id;
    memcpy(id.internal, d->nccl_id, 128);
    ncclComm_t comm;
    GSAP_NCCL(nccl_api()->CommInitRank(&comm, d->nranks, id, d->rank));
    c.nccl_comm = comm;
    c.nranks = d->nranks;
    c.rank = d->rank;
}

void comm_destroy(Ctx &c) {
    if (c.nccl_comm) nccl_api()->CommDestroy((ncclComm_t)c.nccl_comm);
    c.nccl_comm = nullptr;
}

// in place: rank g's block of count_per_rank elements sits at recv + g * count_per_rank
void comm_allgather(Ctx &c, void *recv, size_t count_per_rank, int dtype) {
    if (c.nranks <= 1) return;
    const ncclDataType_t t = dtype == 0 ? ncclInt8 : (dtype == 1 ? ncclInt32 : ncclFloat64);
    const size_t esz = dtype == 0 ? 1 : (dtype == 1 ? 4 : 8);
    const char *send = (const char *)recv + (size_t)c.rank * count_per_rank * esz;
    cudaEvent_t ev = nullptr;
    kc_begin(c, c.k_comm, &ev);
    GSAP_NCCL(nccl_api()->AllGather(send, recv, count_per_rank, t, (ncclComm_t)c.nccl_comm, c.stream));
    kc_end(c, c.k_comm, ev, (double)count_per_rank * esz * c.nranks);
}

// variable slices, in place: rank g's cnt[g] elements at buf + off[g] go to
// every rank (one ncclBroadcast rooted at each rank, in one NCCL group: an
// all-gather-v without padding, so the gathered array is contiguous)
void comm_allgatherv(Ctx &c, void *buf, const std::vector<int> &off, const std::vector<int> &cnt, int dtype) {
    if (c.nranks <= 1) return;
    const ncclDataType_t t = dtype == 0 ? ncclInt8 : (dtype == 1 ? ncclInt32 : ncclFloat64);
    const size_t esz = dtype == 0 ? 1 : (dtype == 1 ? 4 : 8);
    cudaEvent_t ev = nullptr;
    kc_begin(c, c.k_comm, &ev);
    NcclApi *api = nccl_api();
    GSAP_NCCL(api->GroupStart());
    size_t bytes = 0;
    for (int g = 0; g < c.nranks; ++g) {
        if (cnt[g] <= 0) continue;
        char *p = (char *)buf + (size_t)off[g] * esz;
        GSAP_NCCL(api->Broadcast(p, p, (size_t)cnt[g], t, g, (ncclComm_t)c.nccl_comm, c.stream));
        bytes += (size_t)cnt[g] * esz;
    }
    GSAP_NCCL(api->GroupEnd());
    kc_end(c, c.k_comm, ev, (double)bytes);
}

// the MOVE batch [first, first + count) cut into G contiguous slices of whole
// APPLY_CHUNK_V chunks (offsets relative to first), balanced by the work of
// each chunk: adjacency entries + a fixed 16 per vertex (SURVEY 8(e):
// edge-balanced cut points rounded to the fixed reduction chunk, so every
// partial sum covers the same vertices for any G).  Same plan on every rank.
void shard_plan(const Ctx &c, int first, int count, int G, std::vector<int> &off, std::vector<int> &cnt) {
    const int CH = APPLY_CHUNK_V;
    const int chunks = (count + CH - 1) / CH;
    auto work = [&](int v0, int v1) {   // adjacency entries + 16 per vertex of [v0, v1)
        return (long long)(c.h_rowptr[v1] - c.h_rowptr[v0]) + (c.h_cscptr[v1] - c.h_cscptr[v0]) +
               16LL * (v1 - v0);
    };
    const long long total = work(first, first + count);
    off.assign(G, count);
    cnt.assign(G, 0);
    int k = 0;             // next chunk
    long long done = 0;    // work of chunks [0, k)
    for (int g = 0; g < G; ++g) {
        const int k0 = k;
        if (g == G - 1) {
            k = chunks;
        } else {
            const long long target = total * (g + 1) / G;
            while (k < chunks) {
                const int v0 = first + k * CH, v1 = first + std::min(count, (k + 1) * CH);
                const long long wk = work(v0, v1);
                // take chunk k if that ends at or below the target, or overshoots it by less than stopping undershoots
                if (done + wk <= target || done + wk - target < target - done) {
                    done += wk;
                    ++k;
                } else {
                    break;
                }
            }
        }
        off[g] = std::min(count, k0 * CH);
        cnt[g] = std::min(count, k * CH) - off[g];
    }
}

void shard_slice(int n, int chunk, int G, int g, int *first, int *count, int *per_rank) {
    const long long chunks = ((long long)n + chunk - 1) / chunk;
    const long long per = (chunks + G - 1) / G;
    const long long f = std::min<long long>((long long)g * per * chunk, n);
    const long long e = std::min<long long>((long long)(g + 1) * per * chunk, n);
    *first = (int)f;
    *count = (int)(e - f);
    *per_rank = (int)(per * chunk);
}

}  // namespace gsap
