// bp.cu -- rows a3-a6 of the hot path: one NetAlignBP iteration,
// Alg. 2 lines 9-16, as three kernels:
//
//   k_top2    per-vertex (max1, max2) of y^p over A rows of L and of z^p over
//             B columns (the "othermaxrow/othermaxcol" reductions, :164-165,
//             defined at :203)
//   k_edge    per edge: d = alpha w + sum_f F_ef (line 10), y^c = d - omc(z^p),
//             z^c = d - omr(y^p) (lines 11-12), u = y^c + z^c - d (the diagonal
//             of line 13), damping of y, z (lines 14-15)
//   k_square  per unordered square {e < f}: the pair (S^p_ef, S^p_fe) is read
//             once, F_ef = clamp(beta + S^p_fe), F_fe = clamp(beta + S^p_ef)
//             (line 9), S^c = u - F (line 13), damping (line 16), and the
//             NEXT iteration's F row sums are accumulated from the new pair
//             (fusion across iterations; the paper fuses only lines 9-10,
//             Listing 1, :225-262, :266).
//
// Jacobi semantics (reading Z22): k_top2 reads only old y^p, z^p before
// k_edge overwrites them; k_square reads each pair before writing it, and
// both values of a pair live in the same 16 bytes, so no entry ever sees a
// partially updated S^p.
//
// Arithmetic: compiled with --fmad=false; every product and sum is rounded as
// written, like the oracle (-ffp-contract=off).  The only difference from the
// oracle in fast mode is the F row sum: an order-independent fixed-point
// integer sum (exact per term to 2^-fp_bits, deterministic, see DESIGN.md
// "Row sums"); CUALIGN_FLAG_EXACT sums in the oracle's order instead.
#include "internal.cuh"

#include <math.h>

namespace cualign {

namespace {

#define FULL_MASK 0xffffffffu

constexpr int TOP2_G = 8; // lanes per vertex in k_top2

__device__ __forceinline__ void top2_push(double &m1, double &m2, double v)
{
    if (v > m1) {
        m2 = m1;
        m1 = v;
    } else if (v > m2) {
        m2 = v;
    }
}

__device__ __forceinline__ void top2_merge(double &m1, double &m2, double b1, double b2)
{
    const double hi = (b1 > m1) ? b1 : m1;
    const double lo = (b1 > m1) ? m1 : b1;
    double r2 = (b2 > m2) ? b2 : m2;
    r2 = (lo > r2) ? lo : r2;
    m1 = hi;
    m2 = r2;
}

// om(e) from the (max1, max2) of e's row/column (reading Z4)
template <bool LITERAL>
__device__ __forceinline__ double othermax(double v, double2 t)
{
    const double o = (v == t.x) ? t.y : t.x;
    if (LITERAL) return (o == -INFINITY) ? 0.0 : o;
    return (o > 0.0) ? o : 0.0;
}

__device__ __forceinline__ double clamp_beta(double x, double beta)
{
    // bound_{0,beta} exactly as Listing 1 (:247-254)
    double v = x;
    if (v < 0.0) v = 0.0;
    if (v > beta) v = beta;
    return v;
}

__global__ void __launch_bounds__(256)
k_top2(int32_t nA, int32_t nB, const int64_t *__restrict__ Arow, const int64_t *__restrict__ Bptr,
       const int32_t *__restrict__ Bedge, const double *__restrict__ yp, const double *__restrict__ zp,
       double2 *__restrict__ Atop, double2 *__restrict__ Btop)
{
    constexpr int VPW = 32 / TOP2_G;
    const int lane = threadIdx.x & 31;
    const int sub = lane % TOP2_G;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t N = (int64_t)nA + nB;
    for (int64_t base = warp * VPW; base < N; base += nwarps * VPW) {
        const int64_t v = base + lane / TOP2_G;
        double m1 = -INFINITY, m2 = -INFINITY;
        if (v < nA) {
            const int64_t lo = Arow[v], hi = Arow[v + 1];
            for (int64_t x = lo + sub; x < hi; x += TOP2_G) top2_push(m1, m2, yp[x]);
        } else if (v < N) {
            const int64_t b = v - nA;
            const int64_t lo = Bptr[b], hi = Bptr[b + 1];
            for (int64_t x = lo + sub; x < hi; x += TOP2_G) top2_push(m1, m2, zp[Bedge[x]]);
        }
#pragma unroll
        for (int off = TOP2_G / 2; off >= 1; off >>= 1) {
            const double b1 = __shfl_xor_sync(FULL_MASK, m1, off);
            const double b2 = __shfl_xor_sync(FULL_MASK, m2, off);
            top2_merge(m1, m2, b1, b2);
        }
        if (sub == 0) {
            if (v < nA) Atop[v] = make_double2(m1, m2);
            else if (v < N) Btop[v - nA] = make_double2(m1, m2);
        }
    }
}

template <bool EXACT, bool LITERAL>
__global__ void __launch_bounds__(256)
k_edge(int64_t m, const int32_t *__restrict__ La, const int32_t *__restrict__ Lb,
       const double *__restrict__ w, double alpha, double g, double hh, double fp_inv,
       unsigned long long *__restrict__ tacc, const double *__restrict__ texact,
       const double2 *__restrict__ Atop, const double2 *__restrict__ Btop, double *__restrict__ yp,
       double *__restrict__ zp, double *__restrict__ yc, double *__restrict__ zc,
       double *__restrict__ d, double *__restrict__ u)
{
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m;
         e += (int64_t)gridDim.x * blockDim.x) {
        double t;
        if (EXACT) {
            t = texact[e];
        } else {
            const unsigned long long T = tacc[e];
            tacc[e] = 0ull; // ready for this iteration's k_square accumulation
            t = __ull2double_rn(T) * fp_inv;
        }
        const double de = alpha * w[e] + t;                       // line 10
        const double ype = yp[e], zpe = zp[e];
        const double omc = othermax<LITERAL>(zpe, Btop[Lb[e]]);   // line 11
        const double omr = othermax<LITERAL>(ype, Atop[La[e]]);   // line 12
        const double yce = de - omc;
        const double zce = de - omr;
        const double ue = (yce + zce) - de;                       // line 13 diagonal
        yp[e] = g * yce + hh * ype;                               // line 14
        zp[e] = g * zce + hh * zpe;                               // line 15
        yc[e] = yce;
        zc[e] = zce;
        d[e] = de;
        u[e] = ue;
    }
}

// segmented (by sorted key) warp sum, then one atomic per segment
__device__ __forceinline__ void seg_atomic_add(unsigned long long v, int key, int lane,
                                               unsigned long long *dst)
{
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const unsigned long long ov = __shfl_down_sync(FULL_MASK, v, off);
        const int ok = __shfl_down_sync(FULL_MASK, key, off);
        if (lane + off < 32 && ok == key) v += ov;
    }
    const int pk = __shfl_up_sync(FULL_MASK, key, 1);
    const bool head = (lane == 0) || (pk != key);
    if (head && key >= 0 && v) atomicAdd(dst + key, v);
}

// MODE: UPDATE = apply lines 9, 13, 16 to the pair; otherwise only (re)compute
// the F row sums of the current S^p (init, set_state).
template <bool UPDATE, bool EXACT>
__global__ void __launch_bounds__(256)
k_square(int64_t nsq, const int2 *__restrict__ sq_ef, double2 *__restrict__ sq_val,
         const double *__restrict__ u, double beta, double g, double hh, double fp_scale,
         unsigned long long *__restrict__ tacc, const longlong2 *__restrict__ sq_pos,
         double *__restrict__ Ffull)
{
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp * 32; base < nsq; base += nwarps * 32) {
        const int64_t q = base + lane;
        int key = -1 - lane;
        unsigned long long Tef = 0ull;
        if (q < nsq) {
            const int2 ef = sq_ef[q];
            double2 v = sq_val[q]; // (S^p_ef, S^p_fe)
            if (UPDATE) {
                const double Fef = clamp_beta(beta + v.y, beta);    // line 9
                const double Ffe = clamp_beta(beta + v.x, beta);
                const double Scef = u[ef.x] - Fef;                  // line 13
                const double Scfe = u[ef.y] - Ffe;
                v.x = g * Scef + hh * v.x;                          // line 16
                v.y = g * Scfe + hh * v.y;
                sq_val[q] = v;
            }
            // F of the next iteration (line 9 at p+1) from the new pair
            const double Nef = clamp_beta(beta + v.y, beta);
            const double Nfe = clamp_beta(beta + v.x, beta);
            if (EXACT) {
                const longlong2 pos = sq_pos[q];
                Ffull[pos.x] = Nef;
                Ffull[pos.y] = Nfe;
            } else {
                const unsigned long long Tfe = __double2ull_rn(Nfe * fp_scale);
                if (Tfe) atomicAdd(tacc + ef.y, Tfe);
                Tef = __double2ull_rn(Nef * fp_scale);
                key = ef.x;
            }
        }
        if (!EXACT) seg_atomic_add(Tef, key, lane, tacc);
    }
}

// exact mode: t_e = sum of F over row e in ascending f starting from 0.0
__global__ void k_rowsum(int64_t m, const int64_t *__restrict__ Srp, const double *__restrict__ Ffull,
                         double *__restrict__ texact)
{
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m;
         e += (int64_t)gridDim.x * blockDim.x) {
        double t = 0.0;
        for (int64_t pos = Srp[e]; pos < Srp[e + 1]; pos++) t = t + Ffull[pos];
        texact[e] = t;
    }
}

__global__ void k_scatter_Sp(int64_t nsq, const double2 *__restrict__ sq_val,
                             const longlong2 *__restrict__ sq_pos, double *__restrict__ Sfull)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq;
         q += (int64_t)gridDim.x * blockDim.x) {
        const longlong2 pos = sq_pos[q];
        const double2 v = sq_val[q];
        Sfull[pos.x] = v.x;
        Sfull[pos.y] = v.y;
    }
}

__global__ void k_gather_Sp(int64_t nsq, double2 *__restrict__ sq_val, const longlong2 *__restrict__ sq_pos,
                            const double *__restrict__ Sfull)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq;
         q += (int64_t)gridDim.x * blockDim.x) {
        const longlong2 pos = sq_pos[q];
        sq_val[q] = make_double2(Sfull[pos.x], Sfull[pos.y]);
    }
}

int square_grid(cualign_bp *h)
{
    // persistent-style grid: 8 resident 256-thread CTAs per SM
    return grid_for(h->nsq, 256, h->num_sms * 8);
}

cualign_status launch_square(cualign_bp *h, bool update, double g, double hh)
{
    const bool exact = (h->flags & CUALIGN_FLAG_EXACT) != 0;
    if (h->nsq > 0) {
        KScope ks(h, CUALIGN_K_SQUARE);
        const int grid = square_grid(h);
        if (update) {
            if (exact)
                k_square<true, true><<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_ef, h->sq_val, h->u, h->beta, g, hh,
                                                                  h->fp_scale, h->tacc, h->sq_pos, h->Ffull);
            else
                k_square<true, false><<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_ef, h->sq_val, h->u, h->beta, g,
                                                                   hh, h->fp_scale, h->tacc, h->sq_pos, h->Ffull);
        } else {
            if (exact)
                k_square<false, true><<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_ef, h->sq_val, h->u, h->beta, g,
                                                                   hh, h->fp_scale, h->tacc, h->sq_pos, h->Ffull);
            else
                k_square<false, false><<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_ef, h->sq_val, h->u, h->beta, g,
                                                                    hh, h->fp_scale, h->tacc, h->sq_pos, h->Ffull);
        }
        CA_CUDA(cudaGetLastError());
    }
    if (exact) {
        KScope ks(h, CUALIGN_K_ROWSUM);
        const int64_t m = h->L.m;
        if (m) k_rowsum<<<grid_for(m, 128, h->num_sms * 16), 128, 0, h->stream>>>(m, h->Srp, h->Ffull, h->texact);
        CA_CUDA(cudaGetLastError());
    }
    return CUALIGN_OK;
}

} // namespace

cualign_status bp_fsum(cualign_bp *h)
{
    if (!(h->flags & CUALIGN_FLAG_EXACT))
        CA_CUDA(cudaMemsetAsync(h->tacc, 0, sizeof(unsigned long long) * (size_t)(h->L.m ? h->L.m : 1), h->stream));
    return launch_square(h, false, 0.0, 1.0);
}

cualign_status bp_iterate(cualign_bp *h, int32_t n)
{
    const bool exact = (h->flags & CUALIGN_FLAG_EXACT) != 0;
    const bool literal = (h->flags & CUALIGN_FLAG_OTHERMAX_LITERAL) != 0;
    const int64_t m = h->L.m;
    for (int32_t k = 0; k < n; k++) {
        const int32_t p = h->p + 1;
        const double g = pow(h->gamma, (double)p); // reading Z2: host fp64 gamma^p
        const double hh = 1.0 - g;
        if (m > 0) {
            {
                KScope ks(h, CUALIGN_K_TOP2);
                const int64_t N = (int64_t)h->L.nA + h->L.nB;
                const int64_t threads = (N + (32 / TOP2_G) - 1) / (32 / TOP2_G) * 32;
                k_top2<<<grid_for(threads, 256, 1 << 30), 256, 0, h->stream>>>(
                    h->L.nA, h->L.nB, h->L.Arow, h->L.Bptr, h->L.Bedge, h->yp, h->zp, h->Atop, h->Btop);
                CA_CUDA(cudaGetLastError());
            }
            {
                KScope ks(h, CUALIGN_K_EDGE);
                const int grid = grid_for(m, 256, 1 << 30);
#define EDGE_ARGS                                                                                    \
    m, h->L.La, h->L.Lb, h->L.w, h->alpha, g, hh, h->fp_inv, h->tacc, h->texact, h->Atop, h->Btop, \
        h->yp, h->zp, h->yc, h->zc, h->d, h->u
                if (exact && literal) k_edge<true, true><<<grid, 256, 0, h->stream>>>(EDGE_ARGS);
                else if (exact) k_edge<true, false><<<grid, 256, 0, h->stream>>>(EDGE_ARGS);
                else if (literal) k_edge<false, true><<<grid, 256, 0, h->stream>>>(EDGE_ARGS);
                else k_edge<false, false><<<grid, 256, 0, h->stream>>>(EDGE_ARGS);
#undef EDGE_ARGS
                CA_CUDA(cudaGetLastError());
            }
            CA_TRY(launch_square(h, true, g, hh));
        }
        h->p = p;
    }
    return CUALIGN_OK;
}

cualign_status bp_scatter_Sp(cualign_bp *h, double *Sfull_dev)
{
    CA_TRY(ensure_sq_pos(h));
    KScope ks(h, CUALIGN_K_STATE);
    if (h->nsq)
        k_scatter_Sp<<<grid_for(h->nsq, 256, h->num_sms * 8), 256, 0, h->stream>>>(h->nsq, h->sq_val, h->sq_pos,
                                                                                  Sfull_dev);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status bp_gather_Sp(cualign_bp *h, const double *Sfull_dev)
{
    CA_TRY(ensure_sq_pos(h));
    KScope ks(h, CUALIGN_K_STATE);
    if (h->nsq)
        k_gather_Sp<<<grid_for(h->nsq, 256, h->num_sms * 8), 256, 0, h->stream>>>(h->nsq, h->sq_val, h->sq_pos,
                                                                                 Sfull_dev);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

} // namespace cualign
