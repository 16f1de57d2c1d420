// shard.cu -- row e of the hot path: the BP iteration sharded
// by contiguous blocks of A vertices (= blocks of canonical L edge ids).  The
// paper runs on one GPU and names multi-GPU as future work.
//
// A shard owns the L edges [e0, e1) (whole A rows, so othermaxrow is local),
// the S rows of those edges (the squares {e<f} with e owned), and the owned
// entries of y^p, z^p, d.  Per iteration the exchanges are:
//   1. B-side top-2: every shard reduces its owned edges per B vertex; the
//      partials are all-gathered and merged (max is exact).
//   2. u: each shard's owned slice is all-gathered (the square pass needs
//      u_f of any f).
//   3. F row sums: each shard accumulates fixed-point partial sums for every
//      edge; the slices are reduce-scattered to their owners.  Integer sums
//      are associative, so the result is bitwise the single-GPU one.
//   Rounding (a7) is sharded (NEXT-1, see match.cu dist_match_*): proposals
//   from the owned A rows, per-round all-reduces of the B-side suitors; the
//   final matching and its evaluation (a8) are then replicated.
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
    ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
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
            api.AllReduce = (decltype(api.AllReduce))dlsym(lib, "ncclAllReduce");
            api.GroupStart = (decltype(api.GroupStart))dlsym(lib, "ncclGroupStart");
            api.GroupEnd = (decltype(api.GroupEnd))dlsym(lib, "ncclGroupEnd");
            api.GetErrorString = (decltype(api.GetErrorString))dlsym(lib, "ncclGetErrorString");
            api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.AllGather && api.Broadcast &&
                     api.Reduce && api.AllReduce && api.GroupStart && api.GroupEnd && api.GetErrorString;
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

enum RedOp { RED_MAX_U64, RED_MIN_I32, RED_SUM_U64 };

struct Exchange {
    virtual ~Exchange() {}
    virtual cualign_status top2(std::vector<cualign_bp *> &S) = 0;
    virtual cualign_status allgather(std::vector<cualign_bp *> &S, double *cualign_bp::*field) = 0;
    virtual cualign_status reduce_t(std::vector<cualign_bp *> &S) = 0;
    // in-place all-reduce of an array of n entries held by every shard
    virtual cualign_status allreduce(std::vector<cualign_bp *> &S, void *(*field)(cualign_bp *), int64_t n,
                                     RedOp op) = 0;
};

__global__ void k_red_max_u64(int64_t n, unsigned long long *dst, const unsigned long long *src)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (src[i] > dst[i]) dst[i] = src[i];
}
__global__ void k_red_min_i32(int64_t n, int32_t *dst, const int32_t *src)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (src[i] < dst[i]) dst[i] = src[i];
}
__global__ void k_red_sum_u64(int64_t n, unsigned long long *dst, const unsigned long long *src)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] += src[i];
}

size_t red_size(RedOp op) { return op == RED_MIN_I32 ? sizeof(int32_t) : sizeof(unsigned long long); }

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
    cualign_status allreduce(std::vector<cualign_bp *> &S, void *(*field)(cualign_bp *), int64_t n,
                             RedOp op) override
    {
        // fold every shard into shard 0 (fixed order), then copy back
        cualign_bp *h = S[0];
        void *dst = field(h);
        const int grid = grid_for(n, 256, h->num_sms * 8);
        for (size_t r = 1; r < S.size() && n; r++) {
            const void *src = field(S[r]);
            if (op == RED_MAX_U64)
                k_red_max_u64<<<grid, 256, 0, h->stream>>>(n, (unsigned long long *)dst, (const unsigned long long *)src);
            else if (op == RED_MIN_I32)
                k_red_min_i32<<<grid, 256, 0, h->stream>>>(n, (int32_t *)dst, (const int32_t *)src);
            else
                k_red_sum_u64<<<grid, 256, 0, h->stream>>>(n, (unsigned long long *)dst, (const unsigned long long *)src);
            CA_CUDA(cudaGetLastError());
        }
        for (size_t r = 1; r < S.size() && n; r++)
            CA_CUDA(cudaMemcpyAsync(field(S[r]), dst, red_size(op) * (size_t)n, cudaMemcpyDeviceToDevice, h->stream));
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
    cualign_status allreduce(std::vector<cualign_bp *> &S, void *(*field)(cualign_bp *), int64_t n,
                             RedOp op) override
    {
        cualign_bp *h = S[0];
        void *buf = field(h);
        if (!n) return CUALIGN_OK;
        const ncclDataType_t t = op == RED_MIN_I32 ? ncclInt32 : ncclUint64;
        const ncclRedOp_t o = op == RED_MAX_U64 ? ncclMax : (op == RED_MIN_I32 ? ncclMin : ncclSum);
        CA_NCCL(AllReduce(buf, buf, (size_t)n, t, o, (ncclComm_t)h->comm, h->stream));
        return CUALIGN_OK;
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
    for (cualign_bp *s : S) CA_TRY(ensure_gh(s, (int64_t)s->p + n));
    for (int32_t k = 0; k < n; k++) {
        for (cualign_bp *s : S) CA_TRY(bp_front_top2(s));
        CA_TRY(X->top2(S));
        for (cualign_bp *s : S) CA_TRY(bp_front_edge(s));
        CA_TRY(X->allgather(S, &cualign_bp::u));
        for (cualign_bp *s : S) CA_TRY(bp_iterate_back(s));
        CA_TRY(X->reduce_t(S));
        for (cualign_bp *s : S) s->p += 1;
    }
    h->p = S[0]->p;
    return CUALIGN_OK;
}

cualign_status shard_round(cualign_bp *h)
{
    std::vector<cualign_bp *> S;
    Exchange *X = exchange_for(h, S);
    const int64_t n2B = 2 * (int64_t)S[0]->L.nB;
    for (cualign_bp *s : S) CA_TRY(dist_match_begin(s));
    int rounds = 0;
    while (true) {
        for (cualign_bp *s : S) CA_TRY(dist_match_local(s));
        CA_TRY(X->allreduce(S, [](cualign_bp *q) -> void * { return q->dist_wxg; }, n2B, RED_MAX_U64));
        for (cualign_bp *s : S) CA_TRY(dist_match_cand(s));
        CA_TRY(X->allreduce(S, [](cualign_bp *q) -> void * { return q->dist_wid; }, n2B, RED_MIN_I32));
        for (cualign_bp *s : S) CA_TRY(dist_match_update(s));
        CA_TRY(X->allreduce(S, [](cualign_bp *q) -> void * { return q->dist_cnt; }, 1, RED_SUM_U64));
        unsigned long long active = 0;
        CA_CUDA(cudaMemcpyAsync(&active, S[0]->dist_cnt, sizeof(active), cudaMemcpyDeviceToHost, S[0]->stream));
        CA_CUDA(cudaStreamSynchronize(S[0]->stream));
        rounds++;
        if (!active) break;
        if (rounds > (1 << 24)) {
            set_error("sharded rounding did not converge");
            return CUALIGN_ECUDA;
        }
    }
    for (cualign_bp *s : S) {
        s->dist_rounds = rounds;
        CA_TRY(dist_match_finish(s));
    }
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
