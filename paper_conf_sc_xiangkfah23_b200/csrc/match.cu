// match.cu -- rows a7 (rounding by 1/2-approximate matching) and a8
// (evaluate + best) of the hot path: Alg. 2 lines 17-24.
//
// Matching: the locally-dominant algorithm (Preis [24]) as
// synchronous pointer rounds inside ONE persistent cooperative kernel that
// matches y^c and z^c at the same time (two independent instances):
//   init  every vertex (A and B side) points at its heaviest eligible
//         neighbour under the strict order (x desc, edge id asc) (readings
//         Z6, Z7) -- Phase 1's "candidate mate";
//   M     an A vertex whose candidate's B endpoint points back is matched
//         (a locally dominant edge); no atomics: a B vertex has exactly one
//         candidate, so at most one A vertex can claim it;
//   R     unmatched vertices whose candidate endpoint got matched re-point
//         (Phase 2's "those neighbors will have to find new candidates");
//   repeat until a round matches nothing.  grid.sync() separates phases, so
//   the paper's Q_C / Q_N queues are not needed.  Under a strict total order
//   the result is exactly the greedy matching (pin P9), so it is bit-exact
//   against the oracle for identical message vectors.
// Evaluate: weight(M) over the original w (Z9), overlap(M) = x'Sx/2 counted
// on the square layout (each square {e<f} stored once at e), score = alpha w
// + beta overlap (Eq. 1, :64-72), M_y wins ties, best on a strict > (Z8).
#include "internal.cuh"

#include <cooperative_groups.h>

namespace cg = cooperative_groups;

namespace cualign {

namespace {

struct MatchParams {
    int32_t nA, nB;
    int ninst;
    int max_rounds;
    const int32_t *La, *Lb;
    const int64_t *Arow, *Bptr;
    const int32_t *Bedge;
    const double *x[2];
    int32_t *candA, *candB, *mateA, *mateB;
    RoundDev *rd;
    // evaluate
    int evaluate, exact;
    const double *w;
    const int64_t *sq_rp;
    const int2 *sq_ef;
    double alpha, beta;
    double *partial_w;
    int32_t *best_mate;
    int32_t p;
};

__device__ __forceinline__ bool better(double xa, int ea, double xb, int eb)
{
    return eb < 0 || xa > xb || (xa == xb && ea < eb);
}

__device__ int cand_A(const MatchParams &P, int k, int a)
{
    const double *x = P.x[k];
    const int32_t *mB = P.mateB + (int64_t)k * P.nB;
    int best = -1;
    double bx = 0.0;
    const int64_t hi = P.Arow[a + 1];
    for (int64_t e = P.Arow[a]; e < hi; e++) {
        const double xe = x[e];
        if (!(xe > 0.0)) continue;
        if (mB[P.Lb[e]] >= 0) continue;
        if (better(xe, (int)e, bx, best)) {
            best = (int)e;
            bx = xe;
        }
    }
    return best;
}

__device__ int cand_B(const MatchParams &P, int k, int b)
{
    const double *x = P.x[k];
    const int32_t *mA = P.mateA + (int64_t)k * P.nA;
    int best = -1;
    double bx = 0.0;
    const int64_t hi = P.Bptr[b + 1];
    for (int64_t j = P.Bptr[b]; j < hi; j++) {
        const int e = P.Bedge[j];
        const double xe = x[e];
        if (!(xe > 0.0)) continue;
        if (mA[P.La[e]] >= 0) continue;
        if (better(xe, e, bx, best)) {
            best = e;
            bx = xe;
        }
    }
    return best;
}

template <class T>
__device__ T block_sum(T v, T *smem)
{
    // deterministic tree: warp shuffles, then warp 0 over the warp sums
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) v += __shfl_down_sync(0xffffffffu, v, off);
    __syncthreads();
    if (lane == 0) smem[wid] = v;
    __syncthreads();
    const int nw = (blockDim.x + 31) >> 5;
    T r = 0;
    if (wid == 0) {
        r = (lane < nw) ? smem[lane] : (T)0;
#pragma unroll
        for (int off = 16; off >= 1; off >>= 1) r += __shfl_down_sync(0xffffffffu, r, off);
    }
    return r; // valid in thread 0
}

__global__ void __launch_bounds__(256) k_match(MatchParams P)
{
    cg::grid_group grid = cg::this_grid();
    __shared__ double sd[32];
    __shared__ unsigned long long su[32];
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    const int64_t nA = P.nA, nB = P.nB;
    const int64_t NV = nA + nB;
    RoundDev *rd = P.rd;

    if (tid == 0) {
        for (int k = 0; k < 2; k++) {
            rd->flag[0][k] = rd->flag[1][k] = 0;
            rd->rounds[k] = 0;
            rd->overlap[k] = 0;
            rd->card[k] = 0;
            rd->weight[k] = 0.0;
        }
    }
    for (int64_t v = tid; v < P.ninst * NV; v += nthr) {
        const int k = (int)(v / NV);
        const int64_t r = v - k * NV;
        if (r < nA) P.mateA[k * nA + r] = -1;
        else P.mateB[k * nB + (r - nA)] = -1;
    }
    grid.sync();
    // Phase 1: candidate mates among all (unmatched) vertices
    for (int64_t v = tid; v < P.ninst * NV; v += nthr) {
        const int k = (int)(v / NV);
        const int64_t r = v - k * NV;
        if (r < nA) P.candA[k * nA + r] = cand_A(P, k, (int)r);
        else P.candB[k * nB + (r - nA)] = cand_B(P, k, (int)(r - nA));
    }
    grid.sync();
    for (int round = 0; round < P.max_rounds; round++) {
        const int par = round & 1;
        // M: locally dominant edges
        for (int64_t v = tid; v < P.ninst * nA; v += nthr) {
            const int k = (int)(v / nA);
            const int64_t a = v - k * nA;
            if (P.mateA[k * nA + a] >= 0) continue;
            const int e = P.candA[k * nA + a];
            if (e < 0) continue;
            const int b = P.Lb[e];
            if (P.candB[k * nB + b] == e) {
                P.mateA[k * nA + a] = e;
                P.mateB[k * nB + b] = e;
                *(volatile unsigned int *)&rd->flag[par][k] = 1u;
            }
        }
        grid.sync();
        const unsigned int f0 = *(volatile unsigned int *)&rd->flag[par][0];
        const unsigned int f1 = *(volatile unsigned int *)&rd->flag[par][1];
        if (f0 == 0u && f1 == 0u) break;
        if (tid == 0) {
            rd->flag[par ^ 1][0] = 0u;
            rd->flag[par ^ 1][1] = 0u;
            rd->rounds[0] += (int)f0;
            rd->rounds[1] += (int)f1;
        }
        // R: re-point vertices whose candidate endpoint was just matched
        for (int64_t v = tid; v < P.ninst * NV; v += nthr) {
            const int k = (int)(v / NV);
            const int64_t r = v - k * NV;
            if (r < nA) {
                if (P.mateA[k * nA + r] >= 0) continue;
                const int e = P.candA[k * nA + r];
                if (e < 0 || P.mateB[k * nB + P.Lb[e]] < 0) continue;
                P.candA[k * nA + r] = cand_A(P, k, (int)r);
            } else {
                const int64_t b = r - nA;
                if (P.mateB[k * nB + b] >= 0) continue;
                const int e = P.candB[k * nB + b];
                if (e < 0 || P.mateA[k * nA + P.La[e]] < 0) continue;
                P.candB[k * nB + b] = cand_B(P, k, (int)b);
            }
        }
        grid.sync();
    }
    if (!P.evaluate) return;

    // a8: evaluate both matchings
    for (int k = 0; k < P.ninst; k++) {
        double wsum = 0.0;
        unsigned long long ov = 0, card = 0;
        const int32_t *mA = P.mateA + (int64_t)k * nA;
        for (int64_t a = tid; a < nA; a += nthr) {
            const int e = mA[a];
            if (e < 0) continue;
            wsum += P.w[e];
            card++;
            const int64_t hi = P.sq_rp[e + 1];
            for (int64_t q = P.sq_rp[e]; q < hi; q++) {
                const int f = P.sq_ef[q].y;
                if (mA[P.La[f]] == f) ov++;
            }
        }
        const double bw = block_sum<double>(wsum, sd);
        if (threadIdx.x == 0) P.partial_w[k * gridDim.x + blockIdx.x] = bw;
        const unsigned long long bo = block_sum<unsigned long long>(ov, su);
        if (threadIdx.x == 0 && bo) atomicAdd(&rd->overlap[k], bo);
        const unsigned long long bc = block_sum<unsigned long long>(card, su);
        if (threadIdx.x == 0 && bc) atomicAdd(&rd->card[k], bc);
    }
    grid.sync();
    if (blockIdx.x == 0) {
        double wk[2] = {0.0, 0.0};
        for (int k = 0; k < P.ninst; k++) {
            if (P.exact) {
                // oracle order: ascending edge id == ascending A vertex
                if (threadIdx.x == 0) {
                    double s = 0.0;
                    const int32_t *mA = P.mateA + (int64_t)k * nA;
                    for (int64_t a = 0; a < nA; a++)
                        if (mA[a] >= 0) s = s + P.w[mA[a]];
                    wk[k] = s;
                }
            } else {
                double s = 0.0;
                for (int i = threadIdx.x; i < (int)gridDim.x; i += blockDim.x) s += P.partial_w[k * gridDim.x + i];
                s = block_sum<double>(s, sd);
                if (threadIdx.x == 0) wk[k] = s;
            }
        }
        if (threadIdx.x == 0) {
            cualign_round_info &I = rd->info;
            const unsigned long long ov0 = *(volatile unsigned long long *)&rd->overlap[0];
            const unsigned long long ov1 = *(volatile unsigned long long *)&rd->overlap[1];
            const unsigned long long c0 = *(volatile unsigned long long *)&rd->card[0];
            const unsigned long long c1 = *(volatile unsigned long long *)&rd->card[1];
            I.iter = P.p;
            I.weight_y = wk[0];
            I.weight_z = wk[1];
            I.overlap_y = (int64_t)ov0;
            I.overlap_z = (int64_t)ov1;
            I.card_y = (int32_t)c0;
            I.card_z = (int32_t)c1;
            I.score_y = P.alpha * wk[0] + P.beta * (double)(int64_t)ov0;
            I.score_z = P.alpha * wk[1] + P.beta * (double)(int64_t)ov1;
            I.rounds_y = rd->rounds[0];
            I.rounds_z = rd->rounds[1];
            const int src = (I.score_y >= I.score_z) ? 0 : 1;
            I.source = src;
            I.score = src ? I.score_z : I.score_y;
            I.improved = 0;
            if (I.score > rd->best_score) {
                rd->best_score = I.score;
                rd->best_iter = P.p;
                I.improved = 1;
            }
            I.best_score = rd->best_score;
            I.best_iter = rd->best_iter;
            rd->improved = I.improved;
            rd->source = src;
        }
    }
    grid.sync();
    if (*(volatile int *)&rd->improved) {
        const int src = *(volatile int *)&rd->source;
        const int32_t *mA = P.mateA + (int64_t)src * nA;
        for (int64_t a = tid; a < nA; a += nthr) P.best_mate[a] = mA[a];
    }
}

cualign_status launch_match(cualign_bp *h, MatchParams &P)
{
    KScope ks(h, CUALIGN_K_MATCH);
    void *args[] = {&P};
    CA_CUDA(cudaLaunchCooperativeKernel((void *)k_match, dim3(h->match_grid), dim3(h->match_block), args, 0,
                                        h->stream));
    return CUALIGN_OK;
}

MatchParams base_params(cualign_bp *h)
{
    MatchParams P{};
    P.nA = h->L.nA;
    P.nB = h->L.nB;
    P.max_rounds = (int)((int64_t)h->L.nA + h->L.nB + 4 > (1 << 30) ? (1 << 30) : (int64_t)h->L.nA + h->L.nB + 4);
    P.La = h->L.La;
    P.Lb = h->L.Lb;
    P.Arow = h->L.Arow;
    P.Bptr = h->L.Bptr;
    P.Bedge = h->L.Bedge;
    P.candA = h->candA;
    P.candB = h->candB;
    P.mateA = h->mateA;
    P.mateB = h->mateB;
    P.rd = h->rd;
    return P;
}

} // namespace

cualign_status match_setup(cualign_bp *h)
{
    const size_t nA = (size_t)h->L.nA, nB = (size_t)h->L.nB;
    CA_TRY(dalloc(h, &h->candA, 2 * nA + 1));
    CA_TRY(dalloc(h, &h->candB, 2 * nB + 1));
    CA_TRY(dalloc(h, &h->mateA, 2 * nA + 1));
    CA_TRY(dalloc(h, &h->mateB, 2 * nB + 1));
    CA_TRY(dalloc(h, &h->best_mate, nA + 1));
    CA_TRY(dalloc(h, &h->rd, 1));
    CA_CUDA(cudaMemsetAsync(h->rd, 0, sizeof(RoundDev), h->stream));
    CA_CUDA(cudaMemsetAsync(h->best_mate, 0xff, sizeof(int32_t) * (nA + 1), h->stream));
    int occ = 0;
    CA_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_match, h->match_block, 0));
    if (occ < 1) occ = 1;
    int64_t want = ((int64_t)2 * (nA + nB) + h->match_block - 1) / h->match_block;
    int64_t cap = (int64_t)occ * h->num_sms;
    h->match_grid = (int)(want < 1 ? 1 : (want > cap ? cap : want));
    CA_TRY(dalloc(h, &h->partial_w, (size_t)2 * h->match_grid));
    return CUALIGN_OK;
}

cualign_status match_round(cualign_bp *h)
{
    MatchParams P = base_params(h);
    const bool damped = (h->flags & CUALIGN_FLAG_ROUND_DAMPED) != 0;
    P.ninst = 2;
    P.x[0] = damped ? h->yp : h->yc;
    P.x[1] = damped ? h->zp : h->zc;
    P.evaluate = 1;
    P.exact = (h->flags & CUALIGN_FLAG_EXACT) ? 1 : 0;
    P.w = h->L.w;
    P.sq_rp = h->sq_rp;
    P.sq_ef = h->sq_ef;
    P.alpha = h->alpha;
    P.beta = h->beta;
    P.partial_w = h->partial_w;
    P.best_mate = h->best_mate;
    P.p = h->p;
    return launch_match(h, P);
}

cualign_status match_standalone(cualign_bp *h, const double *x_dev, int32_t *rounds)
{
    MatchParams P = base_params(h);
    P.ninst = 1;
    P.x[0] = x_dev;
    P.x[1] = x_dev;
    P.evaluate = 0;
    CA_TRY(launch_match(h, P));
    if (rounds) {
        RoundDev r;
        CA_CUDA(cudaMemcpyAsync(&r, h->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream));
        *rounds = r.rounds[0];
    }
    return CUALIGN_OK;
}

} // namespace cualign
