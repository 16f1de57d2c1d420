// shard.cu -- row e of the hot path: the BP iteration sharded
// by contiguous blocks of A vertices (= blocks of canonical L edge ids).  The
// paper runs on one GPU and names multi-GPU as future work.
//
// A shard owns the L edges [e0, e1) (whole A rows, so othermaxrow is local),
// the S rows of those edges (the squares {e<f} with e owned), and the owned
// entries of y^p, z^p, d.  Per iteration the exchanges are:
//   1. B-side top-2: every shard reduces its owned edges per B vertex; the
//      partials are all-gathered and merged (max is exact).
//   2. u halo: a shard's squares {e < f} (e owned) touch f > e only, i.e.
//      edges of the same or higher shards; the owners send exactly the u_f
//      of those remote f (lists exchanged once at init, shard_setup).
//   3. F halo: the F_fe the square pass adds for remote f go back to their
//      owners (packed, scatter-added there).  Integer sums are associative,
//      so the result is bitwise the single-GPU one.
//   Rounding (a7) is sharded (NEXT-1, see match.cu dist_match_*): proposals
//   from the owned A rows, per-round all-reduces of the B-side suitors; the
//   final matching and its evaluation (a8) are then replicated.
// Two transports implement the exchanges: NCCL between processes (one shard
// per GPU, communicator from a unique id broadcast by torch.distributed), and
// an in-process loopback that holds several virtual shards on one device
// (device-to-device copies) so that the sharded path is tested bit for bit
// against the unsharded one on a single GPU.
#include "internal.cuh"

#include <algorithm>
#include <cub/cub.cuh>
#include <dlfcn.h>
#include <thrust/iterator/counting_iterator.h>
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
    ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
    ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
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
            api.AllReduce = (decltype(api.AllReduce))dlsym(lib, "ncclAllReduce");
            api.GroupStart = (decltype(api.GroupStart))dlsym(lib, "ncclGroupStart");
            api.GroupEnd = (decltype(api.GroupEnd))dlsym(lib, "ncclGroupEnd");
            api.GetErrorString = (decltype(api.GetErrorString))dlsym(lib, "ncclGetErrorString");
            api.Send = (decltype(api.Send))dlsym(lib, "ncclSend");
            api.Recv = (decltype(api.Recv))dlsym(lib, "ncclRecv");
            api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.AllGather &&
                     api.AllReduce && api.GroupStart && api.GroupEnd && api.GetErrorString &&
                     api.Send && api.Recv;
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
constexpr int DIST_MAX_BATCH = 16; // merge rounds enqueued per host check (sharded rounding)

// halo helpers
__global__ void k_gather_d(int64_t n, const int32_t *__restrict__ ids, const double *__restrict__ src,
                           double *__restrict__ dst)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = src[ids[i]];
}
__global__ void k_scatter_d(int64_t n, const int32_t *__restrict__ ids, const double *__restrict__ src,
                            double *__restrict__ dst)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[ids[i]] = src[i];
}
__global__ void k_gather_u64(int64_t n, const int32_t *__restrict__ ids, const unsigned long long *__restrict__ src,
                             unsigned long long *__restrict__ dst)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = src[ids[i]];
}
// several requesters may send the same owned id: integer atomics (exact,
// order-independent)
__global__ void k_scatter_add_u64(int64_t n, const int32_t *__restrict__ ids,
                                  const unsigned long long *__restrict__ src, unsigned long long *__restrict__ dst)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (src[i]) atomicAdd(dst + ids[i], src[i]);
}
// 1 = the square reads a remote f (needs the u halo), 0 = owned f only
__global__ void k_remote_key(int64_t nsq, const int2 *__restrict__ sq_ef, int64_t e1, uint8_t *__restrict__ key)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq; q += (int64_t)gridDim.x * blockDim.x)
        key[q] = sq_ef[q].y >= e1 ? 1 : 0;
}

__global__ void k_mark_remote(int64_t nsq, const int2 *__restrict__ sq_ef, int64_t e1, uint8_t *__restrict__ flag)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq; q += (int64_t)gridDim.x * blockDim.x) {
        const int f = sq_ef[q].y;
        if (f >= e1) flag[f] = 1;
    }
}

cualign_status halo_pack_u(cualign_bp *q)
{
    KScope ks(q, CUALIGN_K_OTHER);
    if (q->n_give)
        k_gather_d<<<grid_for(q->n_give, 256, q->num_sms * 8), 256, 0, q->stream>>>(q->n_give, q->halo_give, q->u,
                                                                                 q->hu_out);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}
cualign_status halo_unpack_u(cualign_bp *r)
{
    KScope ks(r, CUALIGN_K_OTHER);
    if (r->n_need)
        k_scatter_d<<<grid_for(r->n_need, 256, r->num_sms * 8), 256, 0, r->stream>>>(r->n_need, r->halo_need, r->hu_in,
                                                                                  r->u);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}
cualign_status halo_pack_t(cualign_bp *r)
{
    KScope ks(r, CUALIGN_K_OTHER);
    if (r->n_need)
        k_gather_u64<<<grid_for(r->n_need, 256, r->num_sms * 8), 256, 0, r->stream>>>(r->n_need, r->halo_need,
                                                                                   r->tacc, r->ht_out);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}
cualign_status halo_unpack_t(cualign_bp *q)
{
    KScope ks(q, CUALIGN_K_OTHER);
    if (q->n_give)
        k_scatter_add_u64<<<grid_for(q->n_give, 256, q->num_sms * 8), 256, 0, q->stream>>>(q->n_give, q->halo_give,
                                                                                        q->ht_in, q->tacc);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

struct Exchange {
    virtual ~Exchange() {}
    // the square-pass halo: u_f to the shards that read it, F sums back
    virtual cualign_status halo_lists(std::vector<cualign_bp *> &S) = 0;
    virtual cualign_status halo_u(std::vector<cualign_bp *> &S) = 0;
    virtual cualign_status halo_t(std::vector<cualign_bp *> &S) = 0;
    virtual cualign_status top2(std::vector<cualign_bp *> &S) = 0;
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

// bytes a shard receives (algorithmic, as a ring moves them) per exchange
int64_t in_top2(const cualign_bp *q) { return (int64_t)(q->world - 1) * q->L.nB * (int64_t)sizeof(double2); }
int64_t in_allreduce(const cualign_bp *q, int64_t n, RedOp op)
{
    return 2 * (int64_t)(q->world - 1) * n * (int64_t)red_size(op) / q->world;
}

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
    cualign_status halo_lists(std::vector<cualign_bp *> &S) override
    {
        const int w = (int)S.size();
        for (int q = 0; q < w; q++) {
            cualign_bp *o = S[(size_t)q];
            o->give_off.assign((size_t)w + 1, 0);
            for (int r = 0; r < w; r++)
                o->give_off[(size_t)r + 1] = o->give_off[(size_t)r] + (S[(size_t)r]->need_off[(size_t)q + 1] -
                                                                       S[(size_t)r]->need_off[(size_t)q]);
            o->n_give = o->give_off[(size_t)w];
            CA_TRY(dalloc(o, &o->halo_give, (size_t)o->n_give + 1));
            for (int r = 0; r < w; r++) {
                cualign_bp *n = S[(size_t)r];
                const int64_t c = n->need_off[(size_t)q + 1] - n->need_off[(size_t)q];
                if (c)
                    CA_CUDA(cudaMemcpyAsync(o->halo_give + o->give_off[(size_t)r], n->halo_need + n->need_off[(size_t)q],
                                            sizeof(int32_t) * (size_t)c, cudaMemcpyDeviceToDevice, o->stream));
            }
        }
        return CUALIGN_OK;
    }
    cualign_status halo_u(std::vector<cualign_bp *> &S) override
    {
        const int w = (int)S.size();
        for (cualign_bp *q : S) CA_TRY(halo_pack_u(q));
        for (int r = 0; r < w; r++) {
            cualign_bp *n = S[(size_t)r];
            CommScope cs(n, n->n_need * (int64_t)sizeof(double));
            for (int q = 0; q < w; q++) {
                cualign_bp *o = S[(size_t)q];
                const int64_t c = n->need_off[(size_t)q + 1] - n->need_off[(size_t)q];
                if (c)
                    CA_CUDA(cudaMemcpyAsync(n->hu_in + n->need_off[(size_t)q], o->hu_out + o->give_off[(size_t)r],
                                            sizeof(double) * (size_t)c, cudaMemcpyDeviceToDevice, n->stream));
            }
        }
        for (cualign_bp *r : S) CA_TRY(halo_unpack_u(r));
        return CUALIGN_OK;
    }
    cualign_status halo_t(std::vector<cualign_bp *> &S) override
    {
        const int w = (int)S.size();
        for (cualign_bp *r : S) CA_TRY(halo_pack_t(r));
        for (int q = 0; q < w; q++) {
            cualign_bp *o = S[(size_t)q];
            CommScope cs(o, o->n_give * (int64_t)sizeof(unsigned long long));
            for (int r = 0; r < w; r++) {
                cualign_bp *n = S[(size_t)r];
                const int64_t c = o->give_off[(size_t)r + 1] - o->give_off[(size_t)r];
                if (c)
                    CA_CUDA(cudaMemcpyAsync(o->ht_in + o->give_off[(size_t)r], n->ht_out + n->need_off[(size_t)q],
                                            sizeof(unsigned long long) * (size_t)c, cudaMemcpyDeviceToDevice,
                                            o->stream));
            }
        }
        for (cualign_bp *q : S) {
            CA_TRY(halo_unpack_t(q));
            CA_TRY(zero_unowned(q));
        }
        return CUALIGN_OK;
    }
    cualign_status top2(std::vector<cualign_bp *> &S) override
    {
        const int64_t nB = S[0]->L.nB;
        for (cualign_bp *q : S) {
            CommScope cs(q, in_top2(q));
            for (cualign_bp *r : S)
                CA_CUDA(cudaMemcpyAsync(q->Btop_all + (int64_t)r->rank * nB, r->Btop_part, sizeof(double2) * (size_t)nB,
                                        cudaMemcpyDeviceToDevice, q->stream));
            CA_TRY(bp_merge_top2(q));
        }
        return CUALIGN_OK;
    }
    cualign_status allreduce(std::vector<cualign_bp *> &S, void *(*field)(cualign_bp *), int64_t n,
                             RedOp op) override
    {
        // fold every shard into shard 0 (fixed order), then copy back
        cualign_bp *h = S[0];
        for (cualign_bp *q : S) CommScope(q, in_allreduce(q, n, op)); // accounting only
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
    cualign_status halo_lists(std::vector<cualign_bp *> &S) override
    {
        cualign_bp *h = S[0];
        const int w = h->world, me = h->rank;
        // need counts of every rank from every owner: all-gather of [w] int64
        int64_t *cnt_d = nullptr;
        CA_TRY(dalloc(h, &cnt_d, (size_t)w * (size_t)(w + 1)));
        std::vector<int64_t> mine((size_t)w), all((size_t)w * w);
        for (int q = 0; q < w; q++) mine[(size_t)q] = h->need_off[(size_t)q + 1] - h->need_off[(size_t)q];
        CA_CUDA(cudaMemcpyAsync(cnt_d + (size_t)w * w, mine.data(), sizeof(int64_t) * (size_t)w,
                                cudaMemcpyHostToDevice, h->stream));
        CA_NCCL(AllGather(cnt_d + (size_t)w * w, cnt_d, (size_t)w, ncclInt64, (ncclComm_t)h->comm, h->stream));
        CA_CUDA(cudaMemcpyAsync(all.data(), cnt_d, sizeof(int64_t) * (size_t)w * w, cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream));
        h->give_off.assign((size_t)w + 1, 0);
        for (int r = 0; r < w; r++) h->give_off[(size_t)r + 1] = h->give_off[(size_t)r] + all[(size_t)r * w + me];
        h->n_give = h->give_off[(size_t)w];
        CA_TRY(dalloc(h, &h->halo_give, (size_t)h->n_give + 1));
        // the id lists: every rank sends its need segment to each owner
        CA_NCCL(GroupStart());
        for (int q = 0; q < w; q++) {
            const int64_t c = h->need_off[(size_t)q + 1] - h->need_off[(size_t)q];
            if (q != me && c)
                CA_NCCL(Send(h->halo_need + h->need_off[(size_t)q], (size_t)c, ncclInt32, q, (ncclComm_t)h->comm,
                             h->stream));
        }
        for (int r = 0; r < w; r++) {
            const int64_t c = h->give_off[(size_t)r + 1] - h->give_off[(size_t)r];
            if (r != me && c)
                CA_NCCL(Recv(h->halo_give + h->give_off[(size_t)r], (size_t)c, ncclInt32, r, (ncclComm_t)h->comm,
                             h->stream));
        }
        CA_NCCL(GroupEnd());
        return CUALIGN_OK;
    }
    cualign_status halo_u(std::vector<cualign_bp *> &S) override
    {
        cualign_bp *h = S[0];
        const int w = h->world, me = h->rank;
        CA_TRY(halo_pack_u(h));
        {
            CommScope cs(h, h->n_need * (int64_t)sizeof(double));
            CA_NCCL(GroupStart());
            for (int r = 0; r < w; r++) {
                const int64_t c = h->give_off[(size_t)r + 1] - h->give_off[(size_t)r];
                if (r != me && c)
                    CA_NCCL(Send(h->hu_out + h->give_off[(size_t)r], (size_t)c, ncclFloat64, r, (ncclComm_t)h->comm,
                                 h->stream));
            }
            for (int q = 0; q < w; q++) {
                const int64_t c = h->need_off[(size_t)q + 1] - h->need_off[(size_t)q];
                if (q != me && c)
                    CA_NCCL(Recv(h->hu_in + h->need_off[(size_t)q], (size_t)c, ncclFloat64, q, (ncclComm_t)h->comm,
                                 h->stream));
            }
            CA_NCCL(GroupEnd());
        }
        return halo_unpack_u(h);
    }
    cualign_status halo_t(std::vector<cualign_bp *> &S) override
    {
        cualign_bp *h = S[0];
        const int w = h->world, me = h->rank;
        CA_TRY(halo_pack_t(h));
        {
            CommScope cs(h, h->n_give * (int64_t)sizeof(unsigned long long));
            CA_NCCL(GroupStart());
            for (int q = 0; q < w; q++) {
                const int64_t c = h->need_off[(size_t)q + 1] - h->need_off[(size_t)q];
                if (q != me && c)
                    CA_NCCL(Send(h->ht_out + h->need_off[(size_t)q], (size_t)c, ncclUint64, q, (ncclComm_t)h->comm,
                                 h->stream));
            }
            for (int r = 0; r < w; r++) {
                const int64_t c = h->give_off[(size_t)r + 1] - h->give_off[(size_t)r];
                if (r != me && c)
                    CA_NCCL(Recv(h->ht_in + h->give_off[(size_t)r], (size_t)c, ncclUint64, r, (ncclComm_t)h->comm,
                                 h->stream));
            }
            CA_NCCL(GroupEnd());
        }
        CA_TRY(halo_unpack_t(h));
        return zero_unowned(h);
    }
    cualign_status top2(std::vector<cualign_bp *> &S) override
    {
        cualign_bp *h = S[0];
        const int64_t nB = h->L.nB;
        CommScope cs(h, in_top2(h));
        CA_NCCL(AllGather(h->Btop_part, h->Btop_all, (size_t)(2 * nB), ncclFloat64, (ncclComm_t)h->comm,
                              h->stream));
        return bp_merge_top2(h);
    }
    cualign_status allreduce(std::vector<cualign_bp *> &S, void *(*field)(cualign_bp *), int64_t n,
                             RedOp op) override
    {
        cualign_bp *h = S[0];
        void *buf = field(h);
        if (!n) return CUALIGN_OK;
        const ncclDataType_t t = op == RED_MIN_I32 ? ncclInt32 : ncclUint64;
        const ncclRedOp_t o = op == RED_MAX_U64 ? ncclMax : (op == RED_MIN_I32 ? ncclMin : ncclSum);
        CommScope cs(h, in_allreduce(h, n, op));
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

// Stable partition of a shard's squares: those whose f is owned first (the
// square pass over them needs no halo and runs while the u halo is in
// flight), then those with a remote f.  Every result is order-independent
// (integer F sums, per-square arithmetic), so the order changes no bit.  The
// split is rounded down to an even index: the second part's bulk copies need
// 16-byte aligned starts (a local square in the second part only waits).
// S^p is still zero here, so only (e, f) moves.
cualign_status split_squares(cualign_bp *s)
{
    s->nsq_split = -1;
    const int64_t n = s->nsq;
    if (n < 2 || n >= INT32_MAX) return CUALIGN_OK;
    TmpBuf kin, kout, vout, tmp, cnt;
    CA_CUDA(tmalloc(s, kin, (size_t)n));
    CA_CUDA(tmalloc(s, kout, (size_t)n));
    CA_CUDA(tmalloc(s, vout, sizeof(int2) * (size_t)n));
    k_remote_key<<<grid_for(n, 256, s->num_sms * 8), 256, 0, s->stream>>>(n, s->sq_ef, s->e1, (uint8_t *)kin.p);
    CA_CUDA(cudaGetLastError());
    size_t tb = 0;
    const long long *vin = reinterpret_cast<const long long *>(s->sq_ef);
    CA_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, (const uint8_t *)kin.p, (uint8_t *)kout.p, vin,
                                            (long long *)vout.p, (int)n, 0, 1, s->stream));
    CA_CUDA(tmalloc(s, tmp, tb ? tb : 1));
    CA_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tb, (const uint8_t *)kin.p, (uint8_t *)kout.p, vin,
                                            (long long *)vout.p, (int)n, 0, 1, s->stream));
    CA_CUDA(cudaMemcpyAsync(s->sq_ef, vout.p, sizeof(int2) * (size_t)n, cudaMemcpyDeviceToDevice, s->stream));
    // number of local squares = number of zero keys (sum of the keys = remote ones)
    CA_CUDA(tmalloc(s, cnt, sizeof(int64_t)));
    TmpBuf tmp2;
    size_t tb2 = 0;
    CA_CUDA(cub::DeviceReduce::Sum(nullptr, tb2, (const uint8_t *)kin.p, (int64_t *)cnt.p, (int)n, s->stream));
    CA_CUDA(tmalloc(s, tmp2, tb2 ? tb2 : 1));
    CA_CUDA(cub::DeviceReduce::Sum(tmp2.p, tb2, (const uint8_t *)kin.p, (int64_t *)cnt.p, (int)n, s->stream));
    int64_t remote = 0;
    CA_CUDA(cudaMemcpyAsync(&remote, cnt.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s->stream));
    CA_CUDA(cudaStreamSynchronize(s->stream));
    s->nsq_split = ((n - remote) / 2) * 2;
    return pack_squares(s); // the order changed; chunks are also cut at nsq_split
}

// The square-pass halo of every shard: mark the remote f of the owned
// squares, compact them (sorted), split by owner, exchange the lists.
cualign_status shard_setup(cualign_bp *h)
{
    std::vector<cualign_bp *> S;
    Exchange *X = exchange_for(h, S);
    for (cualign_bp *s : S) {
        KScope ks(s, CUALIGN_K_INIT);
        const int64_t m = s->L.m;
        TmpBuf flag, nsel, tmp;
        CA_CUDA(tmalloc(s, flag, (size_t)m + 1));
        CA_CUDA(tmalloc(s, nsel, sizeof(int64_t)));
        CA_CUDA(cudaMemsetAsync(flag.p, 0, (size_t)m + 1, s->stream));
        if (s->nsq)
            k_mark_remote<<<grid_for(s->nsq, 256, s->num_sms * 8), 256, 0, s->stream>>>(s->nsq, s->sq_ef, s->e1,
                                                                                     (uint8_t *)flag.p);
        CA_CUDA(cudaGetLastError());
        CA_TRY(dalloc(s, &s->halo_need, (size_t)m + 1)); // upper bound; the used prefix is n_need
        size_t tb = 0;
        thrust::counting_iterator<int32_t> iota(0);
        CA_CUDA(cub::DeviceSelect::Flagged(nullptr, tb, iota, (const uint8_t *)flag.p, s->halo_need,
                                           (int64_t *)nsel.p, (int)m, s->stream));
        CA_CUDA(tmalloc(s, tmp, tb));
        CA_CUDA(cub::DeviceSelect::Flagged(tmp.p, tb, iota, (const uint8_t *)flag.p, s->halo_need, (int64_t *)nsel.p,
                                           (int)m, s->stream));
        CA_CUDA(cudaMemcpyAsync(&s->n_need, nsel.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s->stream));
        CA_CUDA(cudaStreamSynchronize(s->stream));
        std::vector<int32_t> need((size_t)s->n_need);
        if (s->n_need)
            CA_CUDA(cudaMemcpy(need.data(), s->halo_need, sizeof(int32_t) * (size_t)s->n_need, cudaMemcpyDeviceToHost));
        const int w = s->world;
        s->need_off.assign((size_t)w + 1, 0);
        for (int q = 0; q < w; q++)
            s->need_off[(size_t)q + 1] =
                std::lower_bound(need.begin(), need.end(), (int32_t)std::min<int64_t>(s->bounds[(size_t)q + 1], INT32_MAX)) -
                need.begin();
        s->need_off[(size_t)w] = s->n_need;
        CA_TRY(dalloc(s, &s->hu_in, (size_t)s->n_need + 1));
        CA_TRY(dalloc(s, &s->ht_out, (size_t)s->n_need + 1));
        CA_TRY(split_squares(s));
    }
    CA_TRY(X->halo_lists(S));
    for (cualign_bp *s : S) {
        CA_TRY(dalloc(s, &s->hu_out, (size_t)s->n_give + 1));
        CA_TRY(dalloc(s, &s->ht_in, (size_t)s->n_give + 1));
    }
    return CUALIGN_OK;
}

cualign_status shard_fsum(cualign_bp *h)
{
    std::vector<cualign_bp *> S;
    Exchange *X = exchange_for(h, S);
    for (cualign_bp *s : S) CA_TRY(bp_fsum(s));
    return X->halo_t(S);
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
        // the u halo travels on the exchange stream while the squares whose
        // f is owned run (they read no halo value); the remote-f squares
        // wait for it (SURVEY §8(e) "overlap the exchange with interior rows")
        for (cualign_bp *s : S) {
            CA_CUDA(cudaEventRecord(s->fork_ev[0], s->stream));
            CA_CUDA(cudaStreamWaitEvent(s->cstream, s->fork_ev[0], 0));
        }
        std::vector<cudaStream_t> main_streams;
        for (cualign_bp *s : S) {
            main_streams.push_back(s->stream);
            s->stream = s->cstream;
        }
        const cualign_status hs = X->halo_u(S);
        for (size_t i = 0; i < S.size(); i++) S[i]->stream = main_streams[i];
        CA_TRY(hs);
        for (cualign_bp *s : S) CA_CUDA(cudaEventRecord(s->fork_ev[1], s->cstream));
        for (cualign_bp *s : S) {
            const int64_t split = s->nsq_split >= 0 ? s->nsq_split : 0;
            CA_TRY(bp_iterate_back_range(s, 0, split));
        }
        for (cualign_bp *s : S) {
            CA_CUDA(cudaStreamWaitEvent(s->stream, s->fork_ev[1], 0));
            CA_TRY(bp_iterate_back_range(s, s->nsq_split >= 0 ? s->nsq_split : 0, s->nsq));
        }
        CA_TRY(X->halo_t(S));
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
    // Merge rounds are enqueued in batches; the host reads the all-reduced
    // active count once per batch (a round after convergence changes
    // nothing: no proposer is active, the merges reproduce the global
    // suitors).  The batch grows (2, 4, 8, ...) so that a rounding needing r
    // rounds costs ~log2(r) host round trips and < 2r rounds.  Each shard's
    // count is read into pinned memory on its own stream.
    int rounds = 0, batch = 2;
    while (true) {
        for (int b = 0; b < batch; b++) {
            for (cualign_bp *s : S) CA_TRY(dist_match_local(s));
            CA_TRY(X->allreduce(S, [](cualign_bp *q) -> void * { return q->dist_wxg; }, n2B, RED_MAX_U64));
            for (cualign_bp *s : S) CA_TRY(dist_match_cand(s));
            CA_TRY(X->allreduce(S, [](cualign_bp *q) -> void * { return q->dist_wid; }, n2B, RED_MIN_I32));
            for (cualign_bp *s : S) CA_TRY(dist_match_update(s));
            CA_TRY(X->allreduce(S, [](cualign_bp *q) -> void * { return q->dist_cnt; }, 1, RED_SUM_U64));
            CA_CUDA(cudaMemcpyAsync(S[0]->dist_cnt_host + b, S[0]->dist_cnt, sizeof(unsigned long long),
                                    cudaMemcpyDeviceToHost, S[0]->stream));
        }
        CA_CUDA(cudaStreamSynchronize(S[0]->stream));
        int converged_at = -1;
        for (int b = 0; b < batch && converged_at < 0; b++)
            if (S[0]->dist_cnt_host[b] == 0ull) converged_at = b;
        if (converged_at >= 0) {
            rounds += converged_at + 1; // rounds that did work (the rest were no-ops)
            break;
        }
        rounds += batch;
        if (rounds > (1 << 20)) {
            set_error("sharded rounding: no convergence after %d merge rounds", rounds);
            return CUALIGN_ESTATE;
        }
        batch = std::min(2 * batch, DIST_MAX_BATCH);
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
