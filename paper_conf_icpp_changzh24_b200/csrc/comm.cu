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
        api.CommDestroy = (decltype(api.CommDestroy))dlsym(h, "ncclCommDestroy");
        api.GetErrorString = (decltype(api.GetErrorString))dlsym(h, "ncclGetErrorString");
        ok = api.GetUniqueId && api.CommInitRank && api.AllGather && api.CommDestroy && api.GetErrorString;
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
