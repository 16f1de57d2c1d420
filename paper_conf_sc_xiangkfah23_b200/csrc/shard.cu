// shard.cu -- row e of the hot path: the BP iteration sharded
// by contiguous blocks of A vertices (= blocks of canonical L edge ids).  The
// paper runs on one GPU and names multi-GPU as future work.
//
// A shard owns the L edges [e0, e1) (whole A rows, so othermaxrow is local),
// the S rows of those edges (the squares {e<f} with e owned), and the owned
// entries of y^p, z^p, d.  Per iteration the exchanges are:
//   1. B-side top-2: every shard reduces its owned edges per B vertex; the
//      partials are all-gathered and merged (max is exact).
//   2. u, y^c, z^c: each shard's owned slice is all-gathered (the square pass
//      needs u_f of any f; rounding needs the full y^c, z^c).
//   3. F row sums: each shard accumulates fixed-point partial sums for every
//      edge; the slices are reduce-scattered to their owners.  Integer sums
//      are associative, so the result is bitwise the single-GPU one.
//   Rounding (a7, a8) is replicated on every shard (identical inputs, same
//   deterministic kernels).
// Two transports implement the exchanges: NCCL between processes (one shard
// per GPU, communicator from a unique id broadcast by torch.distributed), and
// an in-process loopback that holds several virtual shards on one device
// (device-to-device copies) so that the sharded path is tested bit for bit
// against the unsharded one on a single GPU.
#include "internal.cuh"

#include <dlfcn.h>
#include <nccl.h>

namespace cualign {

namespace {

// NCCL is resolved at run time (dlopen "libnccl.so.2"): a process that already
// loaded torch gets torch's NCCL, and loading this library never pins an NCCL
// version that torch would then fail to bind against.
struct NcclApi {
    bool tried = false, ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Broadcast)(const void *, void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Reduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, int, ncclComm_t,
                           cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi &nccl()
{
    static NcclApi api;
    if (!api.tried) {
        api.tried = true;
        void *lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!lib) lib = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (lib) {
            api.GetUniqueId = (decltype(api.GetUniqueId))dlsym(lib, "ncclGetUniqueId");
            api.CommInitRank = (decltype(api.CommInitRank))dlsym(lib, "ncclCommInitRank");
            api.CommDestroy = (decltype(api.CommDestroy))dlsym(lib, "ncclCommDestroy");
            api.AllGather = (decltype(api.AllGather))dlsym(lib, "ncclAllGather");
            api.Broadcast = (decltype(api.Broadcast))dlsym(lib, "ncclBroadcast");
            api.Reduce = (decltype(api.Reduce))dlsym(lib, "ncclReduce");
            api.GroupStart = (decltype(api.GroupStart))dlsym(lib, "ncclGroupStart");
            api.GroupEnd = (decltype(api.GroupEnd))dlsym(lib, "ncclGroupEnd");
            api.GetErrorString = (decltype(api.GetErrorString))dlsym(lib, "ncclGetErrorString");
            api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.AllGather && api.Broadcast &&
                     api.Reduce && api.GroupStart && api.GroupEnd && api.GetErrorString;
        }
    }
    return api;
}

#define CA_NCCL(call)                                                                          \
    do {                                                                                       \
        if (!nccl().ok) {                                                                      \
            ::cualign::set_error("NCCL (libnccl.so.2) could not be loaded");                  \
            return CUALIGN_ENCCL;                                                              \
        }                                                                                      \
        ncclResult_t _r = nccl().call;                                                         \
        if (_r != ncclSuccess) {                                                               \
            ::cualign::set_error("%s:%d: nccl%s: %s", __FILE__, __LINE__, #call,               \
                                 nccl().GetErrorString(_r));                                   \
            return CUALIGN_ENCCL;                                                              \
        }                                                                                      \
    } while (0)

struct Exchange {
    virtual ~Exchange() {}
    virtual cualign_status top2(std::vector<cualign_bp *> &S) = 0;
    virtual cualign_status allgather(std::vector<cualign_bp *> &S, double *cualign_bp::*field) = 0;
    virtual cualign_status reduce_t(std::vector<cualign_bp *> &S) = 0;
};

cualign_status zero_unowned(cualign_bp *q)
{
    const int64_t m = q->L.m;
    if (q->e0 > 0) CA_CUDA(cudaMemsetAsync(q->tacc, 0, sizeof(unsigned long long) * (size_t)q->e0, q->stream));
    if (q->e1 < m)
        CA_CUDA(cudaMemsetAsync(q->tacc + q->e1, 0, sizeof(unsigned long long) * (size_t)(m - q->e1), q->stream));
    return CUALIGN_OK;
}

// ---------------------------------------------------------------- loopback
struct Loopback : Exchange {
    cualign_status top2(std::vector<cualign_bp *> &S) override
    {
        const int64_t nB = S[0]->L.nB;
        for (cualign_bp *q : S) {
            for (cualign_bp *r : S)
                CA_CUDA(cudaMemcpyAsync(q->Btop_all + (int64_t)r->rank * nB, r->Btop_part, sizeof(double2) * (size_t)nB,
                                        cudaMemcpyDeviceToDevice, q->stream));
            CA_TRY(bp_merge_top2(q));
        }
        return CUALIGN_OK;
    }
    cualign_status allgather(std::vector<cualign_bp *> &S, double *cualign_bp::*field) override
    {
        for (cualign_bp *r : S) {
            const int64_t n = r->e1 - r->e0;
            if (!n) continue;
            for (cualign_bp *q : S)
                if (q != r)
                    CA_CUDA(cudaMemcpyAsync(q->*field + r->e0, r->*field + r->e0, sizeof(double) * (size_t)n,
                                            cudaMemcpyDeviceToDevice, q->stream));
        }
        return CUALIGN_OK;
    }
    cualign_status reduce_t(std::vector<cualign_bp *> &S) override
    {
        for (cualign_bp *r : S) {
            const int64_t n = r->e1 - r->e0;
            if (!n) continue;
            for (cualign_bp *q : S) // fixed order; integer sums are exact anyway
                if (q != r) CA_TRY(bp_add_u64(r, r->tacc + r->e0, q->tacc + r->e0, n));
        }
        for (cualign_bp *q : S) CA_TRY(zero_unowned(q));
        return CUALIGN_OK;
    }
};

// -------------------------------------------------------------------- NCCL
struct Nccl : Exchange {
    cualign_status top2(std::vector<cualign_bp *> &S) override
    {
        cualign_bp *h = S[0];
        const int64_t nB = h->L.nB;
        CA_NCCL(AllGather(h->Btop_part, h->Btop_all, (size_t)(2 * nB), ncclFloat64, (ncclComm_t)h->comm,
                              h->stream));
        return bp_merge_top2(h);
    }
    cualign_status allgather(std::vector<cualign_bp *> &S, double *cualign_bp::*field) override
    {
        // all-gather-v: one in-place broadcast per owner, grouped
        cualign_bp *h = S[0];
        double *buf = h->*field;
        CA_NCCL(GroupStart());
        for (int r = 0; r < h->world; r++) {
            const int64_t off = h->bounds[(size_t)r], n = h->bounds[(size_t)r + 1] - off;
            if (n) CA_NCCL(Broadcast(buf + off, buf + off, (size_t)n, ncclFloat64, r, (ncclComm_t)h->comm, h->stream));
        }
        CA_NCCL(GroupEnd());
        return CUALIGN_OK;
    }
    cualign_status reduce_t(std::vector<cualign_bp *> &S) override
    {
        // reduce-scatter-v: one in-place reduce per owner, grouped
        cualign_bp *h = S[0];
        CA_NCCL(GroupStart());
        for (int r = 0; r < h->world; r++) {
            const int64_t off = h->bounds[(size_t)r], n = h->bounds[(size_t)r + 1] - off;
            if (n)
                CA_NCCL(Reduce(h->tacc + off, h->tacc + off, (size_t)n, ncclUint64, ncclSum, r,
                                   (ncclComm_t)h->comm, h->stream));
        }
        CA_NCCL(GroupEnd());
        return zero_unowned(h);
    }
};

Exchange *exchange_for(cualign_bp *h, std::vector<cualign_bp *> &S)
{
    static thread_local Loopback lb;
    static thread_local Nccl nc;
    if (!h->vshards.empty()) {
        S = h->vshards;
        return &lb;
    }
    S.assign(1, h);
    return &nc;
}

} // namespace

cualign_status shard_fsum(cualign_bp *h)
{
    std::vector<cualign_bp *> S;
    Exchange *X = exchange_for(h, S);
    for (cualign_bp *s : S) CA_TRY(bp_fsum(s));
    return X->reduce_t(S);
}

cualign_status shard_iterate(cualign_bp *h, int32_t n)
{
    std::vector<cualign_bp *> S;
    Exchange *X = exchange_for(h, S);
    const bool damped = (S[0]->flags & CUALIGN_FLAG_ROUND_DAMPED) != 0;
    for (cualign_bp *s : S) CA_TRY(ensure_gh(s, (int64_t)s->p + n));
    for (int32_t k = 0; k < n; k++) {
        for (cualign_bp *s : S) CA_TRY(bp_front_top2(s));
        CA_TRY(X->top2(S));
        for (cualign_bp *s : S) CA_TRY(bp_front_edge(s));
        CA_TRY(X->allgather(S, &cualign_bp::u));
        CA_TRY(X->allgather(S, &cualign_bp::yc));
        CA_TRY(X->allgather(S, &cualign_bp::zc));
        if (damped) {
            CA_TRY(X->allgather(S, &cualign_bp::yp));
            CA_TRY(X->allgather(S, &cualign_bp::zp));
        }
        for (cualign_bp *s : S) CA_TRY(bp_iterate_back(s));
        CA_TRY(X->reduce_t(S));
        for (cualign_bp *s : S) s->p += 1;
    }
    h->p = S[0]->p;
    return CUALIGN_OK;
}

cualign_status shard_round(cualign_bp *h)
{
    if (h->vshards.empty()) return match_round(h);
    for (cualign_bp *s : h->vshards) CA_TRY(match_round(s));
    return CUALIGN_OK;
}

cualign_status nccl_init_comm(cualign_bp *h, const void *unique_id)
{
    ncclUniqueId id;
    memcpy(&id, unique_id, sizeof(id));
    ncclComm_t c = nullptr;
    CA_NCCL(CommInitRank(&c, h->world, id, h->rank));
    h->comm = c;
    return CUALIGN_OK;
}

void nccl_free_comm(cualign_bp *h)
{
    if (h->comm) {
        if (nccl().ok) nccl().CommDestroy((ncclComm_t)h->comm);
        h->comm = nullptr;
    }
}

cualign_status nccl_unique_id(void *out, int32_t len)
{
    if (len < (int32_t)sizeof(ncclUniqueId)) {
        set_error("unique id buffer too small (%d < %zu)", len, sizeof(ncclUniqueId));
        return CUALIGN_EINVAL;
    }
    ncclUniqueId id;
    CA_NCCL(GetUniqueId(&id));
    memcpy(out, &id, sizeof(id));
    return CUALIGN_OK;
}

} // namespace cualign
