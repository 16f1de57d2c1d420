// quality.cu -- NEXT-4 quality harness: the counts behind
// the network-alignment scores the paper reports (NCV-GS^3, PAPER.md:327-333;
// definitions in its refs [18, 20]), see include/cualign_bp.h
// cualign_quality_eval.  Three flat passes:
//   k_q_nodes     per A vertex: aligned / truth / correct counts, image
//                 occupancy of B (injectivity check)
//   k_q_conserved warp per A row: A edges {i < j} whose images are a B edge
//                 (binary search in the sorted B row) -- the overlap of
//                 PAPER.md:60
//   k_q_induced   warp per B row: B edges {u < v} with both ends in the image
// Counts are block-reduced and added to 64-bit counters (exact integers).
#include "internal.cuh"

#include <cub/cub.cuh>

namespace cualign {

namespace {

enum : int { Q_ALIGNED = 0, Q_TRUTH, Q_CORRECT, Q_CONSERVED, Q_INDUCED, Q_NCOUNT };
enum : int { QE_RANGE = 1, QE_NONINJECTIVE = 2, QE_TRUTHRANGE = 4 };

template <int BLOCK>
__device__ __forceinline__ void block_add(unsigned long long v, unsigned long long *dst)
{
    using R = cub::BlockReduce<unsigned long long, BLOCK>;
    __shared__ typename R::TempStorage tmp;
    const unsigned long long s = R(tmp).Sum(v);
    if (threadIdx.x == 0 && s) atomicAdd(dst, s);
}

__global__ void __launch_bounds__(256) k_q_nodes(int32_t nA, int32_t nB, const int32_t *__restrict__ map,
                                                 const int32_t *__restrict__ truth, int32_t *__restrict__ img,
                                                 unsigned long long *__restrict__ cnt, int *__restrict__ err)
{
    unsigned long long aligned = 0, tt = 0, corr = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nA; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t b = map[i];
        if (b >= nB || b < -1) {
            atomicOr(err, QE_RANGE);
            continue;
        }
        if (b >= 0) {
            aligned++;
            if (atomicAdd(img + b, 1) != 0) atomicOr(err, QE_NONINJECTIVE);
        }
        if (truth) {
            const int32_t t = truth[i];
            if (t >= nB || t < -1) atomicOr(err, QE_TRUTHRANGE);
            if (t >= 0) {
                tt++;
                if (b == t) corr++;
            }
        }
    }
    block_add<256>(aligned, cnt + Q_ALIGNED);
    __syncthreads();
    block_add<256>(tt, cnt + Q_TRUTH);
    __syncthreads();
    block_add<256>(corr, cnt + Q_CORRECT);
}

__device__ __forceinline__ bool has_edge(const int64_t *__restrict__ Bp, const int32_t *__restrict__ Bj, int32_t u,
                                         int32_t v)
{
    int64_t lo = Bp[u], hi = Bp[u + 1];
    while (lo < hi) {
        const int64_t mid = lo + ((hi - lo) >> 1);
        const int32_t x = Bj[mid];
        if (x < v) lo = mid + 1;
        else if (x > v) hi = mid;
        else return true;
    }
    return false;
}

// warp per A row i; lanes over the neighbours j > i
__global__ void __launch_bounds__(256) k_q_conserved(int32_t nA, const int64_t *__restrict__ Ap,
                                                     const int32_t *__restrict__ Aj, const int32_t *__restrict__ map,
                                                     const int64_t *__restrict__ Bp, const int32_t *__restrict__ Bj,
                                                     unsigned long long *__restrict__ cnt)
{
    const int lane = threadIdx.x & 31;
    const int64_t w0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long c = 0;
    for (int64_t i = w0; i < nA; i += nw) {
        const int32_t bi = map[i];
        if (bi < 0) continue;
        for (int64_t x = Ap[i] + lane; x < Ap[i + 1]; x += 32) {
            const int32_t j = Aj[x];
            if (j <= (int32_t)i) continue;
            const int32_t bj = map[j];
            if (bj >= 0 && has_edge(Bp, Bj, bi, bj)) c++;
        }
    }
    block_add<256>(c, cnt + Q_CONSERVED);
}

// warp per B row u; lanes over the neighbours v > u
__global__ void __launch_bounds__(256) k_q_induced(int32_t nB, const int64_t *__restrict__ Bp,
                                                   const int32_t *__restrict__ Bj, const int32_t *__restrict__ img,
                                                   unsigned long long *__restrict__ cnt)
{
    const int lane = threadIdx.x & 31;
    const int64_t w0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long c = 0;
    for (int64_t u = w0; u < nB; u += nw) {
        if (!img[u]) continue;
        for (int64_t x = Bp[u] + lane; x < Bp[u + 1]; x += 32) {
            const int32_t v = Bj[x];
            if (v > (int32_t)u && img[v]) c++;
        }
    }
    block_add<256>(c, cnt + Q_INDUCED);
}

double ratio(int64_t a, int64_t b) { return b > 0 ? (double)a / (double)b : 0.0; }

} // namespace

cualign_status quality_eval(cualign_bp *h, const cualign_graph *A, const cualign_graph *B, const int32_t *map_ab,
                            const int32_t *truth, cualign_quality *out)
{
    const bool devp = (h->flags & CUALIGN_FLAG_DEVICE_PTRS) != 0;
    int64_t nnzA = 0, nnzB = 0;
    int64_t *Ap = nullptr, *Bp = nullptr;
    int32_t *Aj = nullptr, *Bj = nullptr;
    CA_TRY(upload_graph(h, A, "graph A", &Ap, &Aj, &nnzA));
    CA_TRY(upload_graph(h, B, "graph B", &Bp, &Bj, &nnzB));
    const int32_t nA = A->n, nB = B->n;
    int32_t *map = nullptr, *tr = nullptr, *img = nullptr;
    unsigned long long *cnt = nullptr;
    int *err = nullptr;
    CA_TRY(dalloc(h, &map, (size_t)nA + 1));
    CA_TRY(dalloc(h, &img, (size_t)nB + 1));
    CA_TRY(dalloc(h, &cnt, Q_NCOUNT));
    CA_TRY(dalloc(h, &err, 1));
    const cudaMemcpyKind kind = devp ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    if (nA) CA_CUDA(cudaMemcpyAsync(map, map_ab, sizeof(int32_t) * (size_t)nA, kind, h->stream));
    if (truth) {
        CA_TRY(dalloc(h, &tr, (size_t)nA + 1));
        if (nA) CA_CUDA(cudaMemcpyAsync(tr, truth, sizeof(int32_t) * (size_t)nA, kind, h->stream));
    }
    CA_CUDA(cudaMemsetAsync(img, 0, sizeof(int32_t) * ((size_t)nB + 1), h->stream));
    CA_CUDA(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * Q_NCOUNT, h->stream));
    CA_CUDA(cudaMemsetAsync(err, 0, sizeof(int), h->stream));
    const int G = h->num_sms * 8;
    {
        KScope ks(h, CUALIGN_K_EVAL);
        if (nA) k_q_nodes<<<grid_for(nA, 256, G), 256, 0, h->stream>>>(nA, nB, map, tr, img, cnt, err);
        CA_CUDA(cudaGetLastError());
    }
    int e = 0;
    CA_CUDA(cudaMemcpyAsync(&e, err, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    if (e) {
        set_error("cualign_quality_eval:%s%s%s", (e & QE_RANGE) ? " map entry out of range" : "",
                  (e & QE_NONINJECTIVE) ? " map not injective (two A vertices share a B vertex)" : "",
                  (e & QE_TRUTHRANGE) ? " truth entry out of range" : "");
        return CUALIGN_EINVAL;
    }
    {
        KScope ks(h, CUALIGN_K_EVAL);
        if (nA) k_q_conserved<<<grid_for((int64_t)nA * 32, 256, G), 256, 0, h->stream>>>(nA, Ap, Aj, map, Bp, Bj, cnt);
        if (nB) k_q_induced<<<grid_for((int64_t)nB * 32, 256, G), 256, 0, h->stream>>>(nB, Bp, Bj, img, cnt);
        CA_CUDA(cudaGetLastError());
    }
    unsigned long long c[Q_NCOUNT];
    CA_CUDA(cudaMemcpyAsync(c, cnt, sizeof(c), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    cualign_quality q{};
    q.n_a = nA;
    q.n_b = nB;
    q.edges_a = nnzA / 2;
    q.edges_b = nnzB / 2;
    q.aligned = (int64_t)c[Q_ALIGNED];
    q.truth_total = (int64_t)c[Q_TRUTH];
    q.correct = (int64_t)c[Q_CORRECT];
    q.conserved = (int64_t)c[Q_CONSERVED];
    q.induced = (int64_t)c[Q_INDUCED];
    q.nc = ratio(q.correct, q.truth_total);
    q.ec = ratio(q.conserved, q.edges_a);
    q.ics = ratio(q.conserved, q.induced);
    q.s3 = ratio(q.conserved, q.edges_a + q.induced - q.conserved);
    q.ncv = ratio(2 * q.aligned, q.n_a + q.n_b);
    q.gs3 = q.s3;
    q.ncv_gs3 = sqrt(q.ncv * q.gs3);
    *out = q;
    return CUALIGN_OK;
}

} // namespace cualign
