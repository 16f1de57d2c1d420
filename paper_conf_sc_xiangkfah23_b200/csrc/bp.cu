// bp.cu -- rows a3-a6 of the hot path: one NetAlignBP iteration,
// Alg. 2 lines 9-16, as three kernels:
//
//   k_top2    per-vertex (max1, max2) of y^p over the A rows of L and of z^p
//             over the B columns -- the inputs of othermaxrow / othermaxcol
//             (:164-165, defined at :203).  8-lane tiles; B columns are cut
//             into chunks of <= 32 entries so hub columns spread over many
//             tiles (the last tile of a column merges its chunks).
//   k_edge    per edge: d = alpha w + sum_f F_ef (line 10), y^c = d - omc(z^p),
//             z^c = d - omr(y^p) (lines 11-12), u = y^c + z^c - d (the diagonal
//             of line 13), damping of y, z (lines 14-15).  Flat and coalesced,
//             EPT edges per thread with all loads issued up front.
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
#include "ptx.cuh"

#include <cooperative_groups.h>
#include <cub/cub.cuh>
#include <math.h>

namespace cg = cooperative_groups;

namespace cualign {

namespace {

#define FULL_MASK 0xffffffffu

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

template <int G, class Tile>
__device__ __forceinline__ void tile_top2(Tile &tile, double &m1, double &m2)
{
#pragma unroll
    for (int off = G / 2; off >= 1; off >>= 1) {
        const double b1 = tile.shfl_xor(m1, off);
        const double b2 = tile.shfl_xor(m2, off);
        top2_merge(m1, m2, b1, b2);
    }
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

constexpr int B_CHUNK = 32;
constexpr int TG_DEFAULT = 2;         // lanes per tile in k_top2 (CUALIGN_TOP2_TG: 1, 2, 4 or 8)

struct Top2Args {
    int64_t nA, nchunks;    // A rows to process (a0 .. a0+nA-1), B chunks
    int64_t a0;
    const int64_t *Arow;
    const int4 *cdesc;     // per B chunk: (start, end) in the incidence, b, first chunk of b (-1: b has one)
    const int64_t *Bcp, *Bptr;
    const int32_t *Bedge;
    const double *yp, *zp;
    double2 *Atop, *Btop, *Bct;
    unsigned int *Bcnt;
};

// TG lanes per tile; each lane keeps B_CHUNK / TG gathers in flight
template <int TG>
__global__ void __launch_bounds__(256) k_top2(Top2Args T)
{
    constexpr int TB_U = B_CHUNK / TG; // gathers per lane per chunk
    pdl_wait();
    auto tile = cg::tiled_partition<TG>(cg::this_thread_block());
    const int lane = tile.thread_rank();
    const int64_t t0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / TG;
    const int64_t nt = ((int64_t)gridDim.x * blockDim.x) / TG;
    for (int64_t t = t0; t < T.nA + T.nchunks; t += nt) {
        double m1 = -INFINITY, m2 = -INFINITY;
        if (t < T.nA) {
            // A row: contiguous edges
            const int64_t a = T.a0 + t;
            const int64_t lo = T.Arow[a], hi = T.Arow[a + 1];
            // TA_U loads per lane in flight before any use (rows are ~k long)
            constexpr int TA_U = B_CHUNK / TG;
            for (int64_t e0 = lo + lane; e0 < hi; e0 += TG * TA_U) {
                double v[TA_U];
#pragma unroll
                for (int j = 0; j < TA_U; j++) v[j] = (e0 + j * TG < hi) ? T.yp[e0 + j * TG] : -INFINITY;
#pragma unroll
                for (int j = 0; j < TA_U; j++) top2_push(m1, m2, v[j]);
            }
            tile_top2<TG>(tile, m1, m2);
            if (lane == 0) T.Atop[a] = make_double2(m1, m2);
        } else {
            // B chunk: gather z^p through the incidence
            const int64_t c = t - T.nA;
            const int4 dsc = __ldg(T.cdesc + c); // one load instead of chunk_b -> Bcp, Bptr
            const int b = dsc.z;
            const int64_t start = dsc.x, end = dsc.y;
            int eidx[TB_U];
#pragma unroll
            for (int j = 0; j < TB_U; j++) {
                const int64_t idx = start + lane + j * TG;
                eidx[j] = idx < end ? __ldg(T.Bedge + idx) : -1;
            }
#pragma unroll
            for (int j = 0; j < TB_U; j++)
                if (eidx[j] >= 0) top2_push(m1, m2, T.zp[eidx[j]]);
            tile_top2<TG>(tile, m1, m2);
            if (lane == 0) {
                if (dsc.w < 0) {
                    T.Btop[b] = make_double2(m1, m2);
                } else {
                    const int64_t c0 = dsc.w, c1 = T.Bcp[b + 1];
                    // hub column: the last chunk to finish merges all chunks
                    T.Bct[c] = make_double2(m1, m2);
                    __threadfence();
                    const unsigned int prev = atomicAdd(T.Bcnt + b, 1u);
                    if (prev == (unsigned int)(c1 - c0 - 1)) {
                        __threadfence();
                        double r1 = -INFINITY, r2 = -INFINITY;
                        for (int64_t cc = c0; cc < c1; cc++) {
                            const double2 o = __ldcg(T.Bct + cc);
                            top2_merge(r1, r2, o.x, o.y);
                        }
                        T.Btop[b] = make_double2(r1, r2);
                        T.Bcnt[b] = 0u; // ready for the next iteration
                    }
                }
            }
        }
    }
}

struct EdgeArgs {
    int64_t e0, e1;      // the edges this handle owns
    const int32_t *La, *Lb;
    const double *w;
    double alpha, fp_inv;
    const double2 *gh;   // gh[p] = (gamma^p, 1 - gamma^p), host-computed (reading Z2)
    const int *p_dev;    // the current iteration p (advanced at its start)
    unsigned long long *tacc;
    const double *texact;
    const double2 *Atop, *Btop;
    double *yp, *zp, *yc, *zc, *d, *u;
};

template <int EPT, bool EXACT, bool LITERAL, int MINB = 1>
__global__ void __launch_bounds__(256, MINB) k_edge(EdgeArgs R)
{
    pdl_wait();
    const int64_t base = R.e0 + (int64_t)blockIdx.x * blockDim.x * EPT + threadIdx.x;
    const double2 ghp = R.gh[*R.p_dev];
    const double g = ghp.x, hh = ghp.y;
    int64_t e[EPT];
    int a[EPT], b[EPT];
    double we[EPT], ype[EPT], zpe[EPT], t[EPT];
#pragma unroll
    for (int j = 0; j < EPT; j++) {
        e[j] = base + (int64_t)j * blockDim.x;
        if (e[j] < R.e1) {
            a[j] = __ldg(R.La + e[j]);
            b[j] = __ldg(R.Lb + e[j]);
            we[j] = __ldg(R.w + e[j]);
            ype[j] = R.yp[e[j]];
            zpe[j] = R.zp[e[j]];
            if (EXACT) {
                t[j] = R.texact[e[j]];
            } else {
                const unsigned long long T = R.tacc[e[j]];
                t[j] = __ull2double_rn(T) * R.fp_inv;
            }
        }
    }
#pragma unroll
    for (int j = 0; j < EPT; j++) {
        if (e[j] >= R.e1) continue;
        const double2 at = __ldg(R.Atop + a[j]);
        const double2 bt = __ldg(R.Btop + b[j]);
        const double de = R.alpha * we[j] + t[j];          // line 10
        const double omc = othermax<LITERAL>(zpe[j], bt);  // line 11
        const double omr = othermax<LITERAL>(ype[j], at);  // line 12
        const double yce = de - omc;
        const double zce = de - omr;
        const double ue = (yce + zce) - de;                // line 13 diagonal
        R.yp[e[j]] = g * yce + hh * ype[j];                // line 14
        R.zp[e[j]] = g * zce + hh * zpe[j];                // line 15
        R.yc[e[j]] = yce;
        R.zc[e[j]] = zce;
        R.d[e[j]] = de;
        R.u[e[j]] = ue;
        if (!EXACT) R.tacc[e[j]] = 0ull; // ready for this iteration's k_square
    }
}

// Warp sum per run of equal keys, then one atomic per run.  Runs are maximal
// stretches of consecutive lanes with the same key; the same key may occur in
// two runs (the squares are sorted by e only inside a tile, so a warp that
// straddles a tile boundary can see e again) and each run is added on its own.
// Run sum = inclusive prefix sum at the run's last lane minus the one before
// its head (u64 arithmetic is exact mod 2^64; the sums stay below 2^62).
__device__ __forceinline__ void seg_atomic_add(unsigned long long v, int key, int lane,
                                               unsigned long long *dst)
{
    unsigned long long incl = v;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const unsigned long long o = __shfl_up_sync(FULL_MASK, incl, off);
        if (lane >= off) incl += o;
    }
    const int kn = __shfl_down_sync(FULL_MASK, key, 1);
    const int kp = __shfl_up_sync(FULL_MASK, key, 1);
    const unsigned last = __ballot_sync(FULL_MASK, lane == 31 || kn != key); // run ends
    const bool head = (lane == 0) || (kp != key);
    const int end = __ffs(last >> lane) - 1 + lane;          // last lane of this lane's run
    const unsigned long long at_end = __shfl_sync(FULL_MASK, incl, end);
    const unsigned long long before = __shfl_sync(FULL_MASK, incl, lane > 0 ? lane - 1 : 0);
    const unsigned long long sum = at_end - (lane > 0 ? before : 0ull);
    if (head && key >= 0 && sum) atomicAdd(dst + key, sum);
}

// UPDATE = apply lines 9, 13, 16 to the pair; otherwise only (re)compute the
// F row sums of the current S^p (init, set_state).
// S^p pair storage: fp64 (double2, default) or fp32 (float2, CUALIGN_FLAG_FP32_S,
// NEXT-3).  Arithmetic is fp64 either way; the fp32 mode rounds the stored
// state once per update and the next iteration's F is taken from the rounded
// (stored) value, so the F sums always describe the state that persists.
template <bool HINTS>
__device__ __forceinline__ double2 load_pair(const double2 *p)
{
    return HINTS ? __ldcs(p) : *p;
}
template <bool HINTS>
__device__ __forceinline__ double2 load_pair(const float2 *p)
{
    const float2 f = HINTS ? __ldcs(p) : *p;
    return make_double2((double)f.x, (double)f.y);
}
template <bool HINTS>
__device__ __forceinline__ double2 store_pair(double2 *p, double2 v)
{
    if (HINTS) __stcs(p, v);
    else *p = v;
    return v;
}
template <bool HINTS>
__device__ __forceinline__ double2 store_pair(float2 *p, double2 v)
{
    const float2 f = make_float2((float)v.x, (float)v.y); // round to nearest
    if (HINTS) __stcs(p, f);
    else *p = f;
    return make_double2((double)f.x, (double)f.y);
}

template <bool UPDATE, bool EXACT, int SQ_U = 2, bool HINTS = true, bool NOATOM = false, class V = double2>
__global__ void __launch_bounds__(256)
k_square(int64_t nsq, const int2 *__restrict__ sq_ef, V *__restrict__ sq_val,
         const double *__restrict__ u, double beta, const double2 *__restrict__ gh,
         const int *__restrict__ p_dev, double fp_scale,
         unsigned long long *__restrict__ tacc, const longlong2 *__restrict__ sq_pos,
         double *__restrict__ Ffull)
{
    // SQ_U warp-rows of 32 squares per pass: all streaming loads of a pass are
    // issued before any use (memory-level parallelism); the square arrays are
    // streamed with evict-first hints (__ldcs / __stcs) so that the per-edge u
    // and the accumulator tacc stay resident in L2.
    // SQ_U, HINTS: template parameters (variants measured in profiles/)
    double g = 0.0, hh = 1.0;
    if (UPDATE) {
        const double2 ghp = gh[*p_dev];
        g = ghp.x;
        hh = ghp.y;
    }
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp * 32 * SQ_U; base < nsq; base += nwarps * 32 * SQ_U) {
        int2 ef[SQ_U];
        double2 v[SQ_U];
        double ue[SQ_U], uf[SQ_U];
#pragma unroll
        for (int j = 0; j < SQ_U; j++) {
            const int64_t q = base + j * 32 + lane;
            if (q < nsq) {
                ef[j] = (HINTS ? __ldcs(sq_ef + q) : sq_ef[q]);
                v[j] = load_pair<HINTS>(sq_val + q); // (S^p_ef, S^p_fe)
            }
        }
        if (UPDATE) {
#pragma unroll
            for (int j = 0; j < SQ_U; j++) {
                const int64_t q = base + j * 32 + lane;
                if (q < nsq) {
                    ue[j] = __ldg(u + ef[j].x);
                    uf[j] = __ldg(u + ef[j].y);
                }
            }
        }
#pragma unroll
        for (int j = 0; j < SQ_U; j++) {
            const int64_t q = base + j * 32 + lane;
            int key = -1 - lane;
            unsigned long long Tef = 0ull;
            if (q < nsq) {
                if (UPDATE) {
                    const double Fef = clamp_beta(beta + v[j].y, beta);    // line 9
                    const double Ffe = clamp_beta(beta + v[j].x, beta);
                    const double Scef = ue[j] - Fef;                       // line 13
                    const double Scfe = uf[j] - Ffe;
                    v[j].x = g * Scef + hh * v[j].x;                       // line 16
                    v[j].y = g * Scfe + hh * v[j].y;
                    v[j] = store_pair<HINTS>(sq_val + q, v[j]);
                }
                // F of the next iteration (line 9 at p+1) from the new pair
                const double Nef = clamp_beta(beta + v[j].y, beta);
                const double Nfe = clamp_beta(beta + v[j].x, beta);
                if (EXACT) {
                    const longlong2 pos = sq_pos[q];
                    Ffull[pos.x] = Nef;
                    Ffull[pos.y] = Nfe;
                } else {
                    const unsigned long long Tfe = __double2ull_rn(Nfe * fp_scale);
                    if (Tfe && !NOATOM) atomicAdd(tacc + ef[j].y, Tfe);
                    Tef = __double2ull_rn(Nef * fp_scale);
                    key = ef[j].x;
                }
            }
            if (!EXACT && !NOATOM) seg_atomic_add(Tef, key, lane, tacc);
        }
    }
}

// ------------------------------------------------ TMA-pipelined square pass
// Same per-square arithmetic as k_square<UPDATE=true, EXACT=false>, but the
// two streams (sq_ef, sq_val) are moved by the bulk-copy engine
// (cp.async.bulk, 1-D TMA) into a ring of shared-memory stages, so the
// streaming reads no longer wait behind the dependent u gathers in the
// consumer warps' scoreboard: one producer lane keeps SQT_STAGES chunks in
// flight per CTA, the consumer warps copy a stage to registers, release it
// (mbarrier arrive) and only then gather u and issue the F-sum atomics.
// The streams carry an evict-first L2 policy (u and tacc stay resident).
constexpr int SQT_CHUNK = 512;            // squares per stage
constexpr int SQT_STAGES = 4;
constexpr int SQT_CWARPS = 8;             // consumer warps; + 1 producer warp
constexpr int SQT_PER_THREAD = SQT_CHUNK / (SQT_CWARPS * 32);

using namespace ptx;

// DYN: chunks taken from a queue (ctr[0], one atomic per chunk by the
// producer lane, STAGES chunks ahead of use) instead of the static stride
// blockIdx + k*grid: a CTA that starts late -- its SM still running the
// rounding branch of a pipelined step -- takes fewer chunks instead of
// finishing last.  The last producer to finish resets the queue (ctr[1]
// counts finished producers).  The chunk id travels with its stage in smem.
template <class V, bool NOATOM = false, bool DYN = false>
__global__ void __launch_bounds__((SQT_CWARPS + 1) * 32)
k_square_tma(int64_t nsq, const int2 *__restrict__ sq_ef, V *__restrict__ sq_val,
             const double *__restrict__ u, double beta, const double2 *__restrict__ gh,
             const int *__restrict__ p_dev, double fp_scale, unsigned long long *__restrict__ tacc,
             unsigned int *__restrict__ ctr)
{
    __shared__ int s_chunk[SQT_STAGES];
    // dynamic shared memory: [full | empty barriers (128 B)] [ef stages] [value stages]
    extern __shared__ __align__(128) unsigned char sq_smem[];
    uint64_t *full = reinterpret_cast<uint64_t *>(sq_smem);
    uint64_t *empty = full + SQT_STAGES;
    int2 (*s_ef)[SQT_CHUNK] = reinterpret_cast<int2 (*)[SQT_CHUNK]>(sq_smem + 128);
    V (*s_val)[SQT_CHUNK] = reinterpret_cast<V (*)[SQT_CHUNK]>(sq_smem + 128 + sizeof(int2) * SQT_STAGES * SQT_CHUNK);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t nchunks = (nsq + SQT_CHUNK - 1) / SQT_CHUNK;
    if (threadIdx.x == 0) {
        for (int s = 0; s < SQT_STAGES; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], SQT_CWARPS);
        }
        fence_mbar_init();
    }
    __syncthreads();
    pdl_wait(); // the barrier setup above overlaps the predecessor's tail
    if (warp == SQT_CWARPS) {
        // producer: one lane issues the bulk copies of this CTA's chunks
        if (lane == 0) {
            const uint64_t policy = policy_evict_first();
            int i = 0;
            for (int64_t c = blockIdx.x;; c += gridDim.x, i++) {
                const int s = i % SQT_STAGES;
                if (i >= SQT_STAGES) mbar_wait(&empty[s], (uint32_t)((i / SQT_STAGES) - 1) & 1u);
                if (DYN) {
                    c = atomicAdd(ctr, 1u);
                    if (c >= nchunks) {
                        s_chunk[s] = -1; // end of queue: released by the arrive
                        mbar_arrive(&full[s]);
                        __threadfence();
                        if (atomicAdd(ctr + 1, 1u) == gridDim.x - 1) {
                            ctr[0] = 0u; // every producer is past its last take
                            ctr[1] = 0u;
                        }
                        break;
                    }
                    s_chunk[s] = (int)c;
                } else if (c >= nchunks) {
                    break;
                }
                const int64_t q0 = c * SQT_CHUNK;
                const int n = (int)((nsq - q0) < SQT_CHUNK ? (nsq - q0) : SQT_CHUNK);
                // 16-byte multiples (the arrays carry 2 elements of padding)
                const uint32_t b_ef = (uint32_t)((n * sizeof(int2) + 15) & ~(size_t)15);
                const uint32_t b_val = (uint32_t)((n * sizeof(V) + 15) & ~(size_t)15);
                mbar_expect_tx(&full[s], b_ef + b_val);
                bulk_load(&s_ef[s][0], sq_ef + q0, b_ef, &full[s], policy);
                bulk_load(&s_val[s][0], sq_val + q0, b_val, &full[s], policy);
            }
        }
        return;
    }
    const double2 ghp = gh[*p_dev];
    const double g = ghp.x, hh = ghp.y;
    const int tid = threadIdx.x; // consumer thread 0 .. SQT_CWARPS*32-1
    int i = 0;
    for (int64_t c = blockIdx.x;; c += gridDim.x, i++) {
        const int s = i % SQT_STAGES;
        if (!DYN && c >= nchunks) break;
        mbar_wait(&full[s], (uint32_t)(i / SQT_STAGES) & 1u);
        if (DYN) {
            c = *(volatile int *)&s_chunk[s];
            if (c < 0) break;
        }
        const int64_t q0 = c * SQT_CHUNK;
        const int n = (int)((nsq - q0) < SQT_CHUNK ? (nsq - q0) : SQT_CHUNK);
        int2 ef[SQT_PER_THREAD];
        double2 v[SQT_PER_THREAD];
#pragma unroll
        for (int j = 0; j < SQT_PER_THREAD; j++) {
            const int r = j * (SQT_CWARPS * 32) + tid; // a warp covers 32 consecutive squares
            if (r < n) {
                ef[j] = s_ef[s][r];
                v[j] = load_pair<false>(&s_val[s][r]);
            }
        }
        // order this warp's generic-proxy reads of the stage before the
        // async-proxy (bulk copy) writes that refill it -- without the fence
        // a refill can land before the LDS has read the stage (measured)
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[s]); // stage may be refilled
        double ue[SQT_PER_THREAD], uf[SQT_PER_THREAD];
#pragma unroll
        for (int j = 0; j < SQT_PER_THREAD; j++) {
            const int r = j * (SQT_CWARPS * 32) + tid;
            if (r < n) {
                ue[j] = __ldg(u + ef[j].x);
                uf[j] = __ldg(u + ef[j].y);
            }
        }
#pragma unroll
        for (int j = 0; j < SQT_PER_THREAD; j++) {
            const int r = j * (SQT_CWARPS * 32) + tid;
            int key = -1 - lane;
            unsigned long long Tef = 0ull;
            if (r < n) {
                const double Fef = clamp_beta(beta + v[j].y, beta);    // line 9
                const double Ffe = clamp_beta(beta + v[j].x, beta);
                const double Scef = ue[j] - Fef;                       // line 13
                const double Scfe = uf[j] - Ffe;
                v[j].x = g * Scef + hh * v[j].x;                       // line 16
                v[j].y = g * Scfe + hh * v[j].y;
                v[j] = store_pair<true>(sq_val + q0 + r, v[j]);
                const double Nef = clamp_beta(beta + v[j].y, beta);   // line 9 at p+1
                const double Nfe = clamp_beta(beta + v[j].x, beta);
                const unsigned long long Tfe = __double2ull_rn(Nfe * fp_scale);
                if (Tfe && !NOATOM) atomicAdd(tacc + ef[j].y, Tfe);
                Tef = __double2ull_rn(Nef * fp_scale);
                key = ef[j].x;
            }
            if (!NOATOM) seg_atomic_add(Tef, key, lane, tacc);
        }
    }
}

// ------------------------------------ packed-index TMA square pass (default)
// k_square_tma over the packed square stream (pack_squares): 4 B of (e, f)
// per square instead of 8 -- 36 B per square moved instead of 40 (18 B per
// nonzero of S instead of 20).  Chunk c = desc[c] = (q0, n, eb, fb) covers
// squares q0 .. q0+n-1 (n <= SQP_CHUNK, chunks cut at tiles and e ranges);
// the producer lane stages the descriptor with the chunk's two streams.  The
// bulk copies start at the 16-byte boundary at or below q0 (offsets ow, ov
// into the stage); the arrays carry 16 bytes of padding for the tails.
constexpr int SQP_STAGES = 4;
template <class V>
constexpr int sqp_val_slack() { return 16 / (int)sizeof(V) - 1; } // elements before q0 in a stage

template <class V>
constexpr size_t square_pk_smem()
{
    return 128 + (size_t)SQP_STAGES * (sizeof(uint32_t) * (SQP_CHUNK + 4) +
                                       sizeof(V) * (SQP_CHUNK + sqp_val_slack<V>() + 1));
}

// PROBE (timing probes of the probe build only, wrong results): bit 0 = no
// F-sum atomics, bit 1 = no u_f gathers (u_e used instead).
// 48 registers (was 51): 4 CTAs per SM then leave 10 K registers, room for
// one 128-thread block of the rounding's chain form (k_suitor_q) beside the
// square pass in the pipelined step instead of after it (bench window on O:
// 1504-1509 -> 1520-1521 it/s; no spills).
template <class V, int PROBE = 0>
__global__ void __maxnreg__(48)
k_square_pk(int64_t c0, int64_t c1, const int4 *__restrict__ desc, const uint32_t *__restrict__ words,
            V *__restrict__ sq_val, const double *__restrict__ u, double beta, const double2 *__restrict__ gh,
            const int *__restrict__ p_dev, double fp_scale, unsigned long long *__restrict__ tacc)
{
    constexpr int WST = SQP_CHUNK + 4;                         // words per stage
    constexpr int VST = SQP_CHUNK + sqp_val_slack<V>() + 1;    // values per stage (16-byte multiple)
    static_assert((WST * 4) % 16 == 0 && (VST * sizeof(V)) % 16 == 0, "stage sizes");
    __shared__ int4 s_desc[SQP_STAGES];
    extern __shared__ __align__(128) unsigned char sq_smem[];
    uint64_t *full = reinterpret_cast<uint64_t *>(sq_smem);
    uint64_t *empty = full + SQP_STAGES;
    uint32_t (*s_w)[WST] = reinterpret_cast<uint32_t (*)[WST]>(sq_smem + 128);
    V (*s_val)[VST] = reinterpret_cast<V (*)[VST]>(sq_smem + 128 + sizeof(uint32_t) * SQP_STAGES * WST);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < SQP_STAGES; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], SQT_CWARPS);
        }
        fence_mbar_init();
    }
    __syncthreads();
    pdl_wait();
    if (warp == SQT_CWARPS) {
        if (lane == 0) {
            const uint64_t policy = policy_evict_first();
            int i = 0;
            int4 dn = (c0 + blockIdx.x < c1) ? __ldg(desc + c0 + blockIdx.x) : make_int4(0, 0, 0, 0);
            for (int64_t c = c0 + blockIdx.x; c < c1; c += gridDim.x, i++) {
                const int s = i % SQP_STAGES;
                const int4 d = dn;
                if (c + gridDim.x < c1) dn = __ldg(desc + c + gridDim.x); // next descriptor in flight
                if (i >= SQP_STAGES) mbar_wait(&empty[s], (uint32_t)((i / SQP_STAGES) - 1) & 1u);
                s_desc[s] = d;
                const int64_t qw = d.x & ~3, qv = d.x & ~(int64_t)sqp_val_slack<V>();
                const uint32_t bw = (uint32_t)(((d.x + d.y - qw) * sizeof(uint32_t) + 15) & ~(size_t)15);
                const uint32_t bv = (uint32_t)(((d.x + d.y - qv) * sizeof(V) + 15) & ~(size_t)15);
                mbar_expect_tx(&full[s], bw + bv); // release: s_desc[s] is visible to the waiters
                bulk_load(&s_w[s][0], words + qw, bw, &full[s], policy);
                bulk_load(&s_val[s][0], sq_val + qv, bv, &full[s], policy);
            }
        }
        return;
    }
    const double2 ghp = gh[*p_dev];
    const double g = ghp.x, hh = ghp.y;
    const int tid = threadIdx.x;
    constexpr int FMASK = (1 << SQP_FBITS) - 1;
    int i = 0;
    for (int64_t c = c0 + blockIdx.x; c < c1; c += gridDim.x, i++) {
        const int s = i % SQP_STAGES;
        mbar_wait(&full[s], (uint32_t)(i / SQP_STAGES) & 1u);
        const int4 d = s_desc[s];
        const int q0 = d.x, n = d.y, eb = d.z, fb = d.w;
        const int ow = q0 & 3, ov = q0 & sqp_val_slack<V>();
        int2 ef[SQT_PER_THREAD];
        double2 v[SQT_PER_THREAD];
#pragma unroll
        for (int j = 0; j < SQT_PER_THREAD; j++) {
            const int r = j * (SQT_CWARPS * 32) + tid;
            if (r < n) {
                const uint32_t w = s_w[s][ow + r];
                ef[j] = make_int2(eb + (int)(w >> SQP_FBITS), fb + (int)(w & FMASK));
                v[j] = load_pair<false>(&s_val[s][ov + r]);
            }
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[s]);
        double ue[SQT_PER_THREAD], uf[SQT_PER_THREAD];
#pragma unroll
        for (int j = 0; j < SQT_PER_THREAD; j++) {
            const int r = j * (SQT_CWARPS * 32) + tid;
            if (r < n) {
                ue[j] = __ldg(u + ef[j].x);
                uf[j] = (PROBE & 2) ? ue[j] : __ldg(u + ef[j].y);
            }
        }
#pragma unroll
        for (int j = 0; j < SQT_PER_THREAD; j++) {
            const int r = j * (SQT_CWARPS * 32) + tid;
            int key = -1 - lane;
            unsigned long long Tef = 0ull;
            if (r < n) {
                const double Fef = clamp_beta(beta + v[j].y, beta);    // line 9
                const double Ffe = clamp_beta(beta + v[j].x, beta);
                const double Scef = ue[j] - Fef;                       // line 13
                const double Scfe = uf[j] - Ffe;
                v[j].x = g * Scef + hh * v[j].x;                       // line 16
                v[j].y = g * Scfe + hh * v[j].y;
                v[j] = store_pair<true>(sq_val + q0 + r, v[j]);
                const double Nef = clamp_beta(beta + v[j].y, beta);   // line 9 at p+1
                const double Nfe = clamp_beta(beta + v[j].x, beta);
                const unsigned long long Tfe = __double2ull_rn(Nfe * fp_scale);
                if (Tfe && !(PROBE & 1)) atomicAdd(tacc + ef[j].y, Tfe);
                Tef = __double2ull_rn(Nef * fp_scale);
                key = ef[j].x;
            }
            if (!(PROBE & 1)) seg_atomic_add(Tef, key, lane, tacc);
        }
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

template <class V>
__global__ void k_scatter_Sp(int64_t nsq, const V *__restrict__ sq_val, const longlong2 *__restrict__ sq_pos,
                             double *__restrict__ Sfull)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq;
         q += (int64_t)gridDim.x * blockDim.x) {
        const longlong2 pos = sq_pos[q];
        const double2 v = load_pair<false>(sq_val + q);
        Sfull[pos.x] = v.x;
        Sfull[pos.y] = v.y;
    }
}

template <class V>
__global__ void k_gather_Sp(int64_t nsq, V *__restrict__ sq_val, const longlong2 *__restrict__ sq_pos,
                            const double *__restrict__ Sfull)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq;
         q += (int64_t)gridDim.x * blockDim.x) {
        const longlong2 pos = sq_pos[q];
        store_pair<false>(sq_val + q, make_double2(Sfull[pos.x], Sfull[pos.y]));
    }
}

__global__ void k_chunk_count(int64_t nB, const int64_t *__restrict__ Bptr, int64_t *__restrict__ cnt)
{
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nB; b += (int64_t)gridDim.x * blockDim.x)
        cnt[b] = (Bptr[b + 1] - Bptr[b] + B_CHUNK - 1) / B_CHUNK;
}

__global__ void k_chunk_fill(int64_t nB, const int64_t *__restrict__ Bcp, const int64_t *__restrict__ Bptr,
                             int4 *__restrict__ cdesc)
{
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nB; b += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c0 = Bcp[b], c1 = Bcp[b + 1], e1 = Bptr[b + 1];
        for (int64_t c = c0; c < c1; c++) {
            const int64_t st = Bptr[b] + (c - c0) * B_CHUNK;
            cdesc[c] = make_int4((int)st, (int)min(st + (int64_t)B_CHUNK, e1), (int)b, c1 - c0 > 1 ? (int)c0 : -1);
        }
    }
}

// Grid-stride kernels run as exactly one wave: (resident CTAs per SM) x SMs,
// capped by the work (a 1.6-wave grid left 40% of the SMs idle in the tail).
int one_wave_grid(cualign_bp *h, const void *fn, int block, int64_t items, int64_t items_per_block)
{
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, block, 0) != cudaSuccess || occ < 1) occ = 1;
    (void)cudaGetLastError();
    return grid_for((items + items_per_block - 1) / items_per_block, 1, occ * h->num_sms);
}

__global__ void k_advance(int *p_dev)
{
    pdl_wait();
    *p_dev += 1;
}

template <bool UPDATE, bool EXACT, int SQ_U, bool HINTS, bool NOATOM, class V>
void square_launch_v(cualign_bp *h, V *vals)
{
    auto fn = k_square<UPDATE, EXACT, SQ_U, HINTS, NOATOM, V>;
    int grid = one_wave_grid(h, (const void *)fn, 256, h->nsq, 256 * SQ_U);
    // leave room for the concurrent rounding branch (graph step): a fraction
    // of the resident CTAs still saturates HBM
    static const double frac = probe_knob("CUALIGN_SQ_FRAC_PCT", 100) / 100.0;
    if (frac > 0.0 && frac < 1.0) grid = (int)(grid * frac) > 0 ? (int)(grid * frac) : 1;
    fn<<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_ef, vals, h->u, h->beta, h->gh_dev, h->p_dev, h->fp_scale, h->tacc,
                                    h->sq_pos, h->Ffull);
}

template <class V>
constexpr size_t square_tma_smem()
{
    return 128 + (sizeof(int2) + sizeof(V)) * SQT_STAGES * SQT_CHUNK;
}

// squares [q0, q1) (q1 < 0: all); q0 even (16-byte aligned bulk copies)
template <class V, bool NOATOM = false, bool DYN = false>
cualign_status square_tma_launch_v(cualign_bp *h, V *vals, int64_t q0 = 0, int64_t q1 = -1)
{
    if (q1 < 0) q1 = h->nsq;
    const int64_t nq = q1 - q0;
    if (nq <= 0) return CUALIGN_OK;
    auto fn = k_square_tma<V, NOATOM, DYN>;
    constexpr size_t smem = square_tma_smem<V>();
    // > 48 KB of dynamic shared memory needs the opt-in attribute, which
    // belongs to the function in the CURRENT device's context: set it on
    // every launch (cheap), so handles on several devices each get it
    CA_CUDA(cudaFuncSetAttribute((const void *)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int block = (SQT_CWARPS + 1) * 32;
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, block, smem) != cudaSuccess || occ < 1) occ = 1;
    (void)cudaGetLastError();
    if (h->sq_ctas > 0 && h->sq_ctas < occ) occ = h->sq_ctas;
    const int64_t nchunks = (nq + SQT_CHUNK - 1) / SQT_CHUNK;
    const int grid = grid_for(nchunks, 1, (int64_t)occ * h->num_sms);
    CA_CUDA(launch_pdl(fn, dim3(grid), dim3(block), smem, h->stream, nq, (const int2 *)(h->sq_ef + q0), vals + q0,
                       (const double *)h->u, h->beta, (const double2 *)h->gh_dev, (const int *)h->p_dev, h->fp_scale,
                       h->tacc, h->sq_ctr));
    return CUALIGN_OK;
}

// chunks [c0, c1) of the packed stream
template <class V>
cualign_status square_pk_launch_v(cualign_bp *h, V *vals, int64_t c0, int64_t c1)
{
    if (c1 <= c0) return CUALIGN_OK;
#ifdef CUALIGN_PROBES
    static const int probe = probe_knob("CUALIGN_SQ_PK_PROBE", 0); // timing probes (wrong results)
    auto fn = probe == 1 ? k_square_pk<V, 1> : (probe == 2 ? k_square_pk<V, 2> : (probe == 3 ? k_square_pk<V, 3> : k_square_pk<V>));
#else
    auto fn = k_square_pk<V>;
#endif
    constexpr size_t smem = square_pk_smem<V>();
    CA_CUDA(cudaFuncSetAttribute((const void *)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int block = (SQT_CWARPS + 1) * 32;
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, block, smem) != cudaSuccess || occ < 1) occ = 1;
    (void)cudaGetLastError();
    if (h->sq_ctas > 0 && h->sq_ctas < occ) occ = h->sq_ctas;
    const int grid = grid_for(c1 - c0, 1, (int64_t)occ * h->num_sms);
    CA_CUDA(launch_pdl(fn, dim3(grid), dim3(block), smem, h->stream, c0, c1, (const int4 *)h->sqp_desc,
                       (const uint32_t *)h->sqp_w, vals, (const double *)h->u, h->beta, (const double2 *)h->gh_dev,
                       (const int *)h->p_dev, h->fp_scale, h->tacc));
    return CUALIGN_OK;
}

// squares [q0, q1) through the packed stream when it covers the range at
// chunk boundaries (all squares, or a sharded part split at nsq_split)
bool square_pk_range(const cualign_bp *h, int64_t q0, int64_t q1, int64_t &c0, int64_t &c1)
{
    if (h->sqp_nchunks <= 0) return false;
    if (q1 < 0) q1 = h->nsq;
    auto chunk_at = [&](int64_t q, int64_t &c) {
        if (q == 0) c = 0;
        else if (q == h->nsq) c = h->sqp_nchunks;
        else if (h->nsq_split > 0 && q == h->nsq_split) c = h->sqp_split_chunk;
        else return false;
        return true;
    };
    return chunk_at(q0, c0) && chunk_at(q1, c1);
}

cualign_status square_tma_launch(cualign_bp *h, int64_t q0 = 0, int64_t q1 = -1)
{
    static const int packed = probe_knob("CUALIGN_SQ_PACKED", 1); // probe build: 0 = int2 index stream
    int64_t c0 = 0, c1 = 0;
    if (packed && square_pk_range(h, q0, q1, c0, c1)) {
        if (h->sq_val32) return square_pk_launch_v(h, h->sq_val32, c0, c1);
        return square_pk_launch_v(h, h->sq_val, c0, c1);
    }
    if (q0 != 0 || q1 >= 0) {
        if (h->sq_val32) return square_tma_launch_v(h, h->sq_val32, q0, q1);
        return square_tma_launch_v(h, h->sq_val, q0, q1);
    }
    // CUALIGN_SQ_DYN (probe build): 1 = chunk queue, 0 = static stride
    static const int dyn = probe_knob("CUALIGN_SQ_DYN", 0);
    if (dyn) {
        if (h->sq_val32) return square_tma_launch_v<float2, false, true>(h, h->sq_val32);
        return square_tma_launch_v<double2, false, true>(h, h->sq_val);
    }
    if (h->sq_val32) return square_tma_launch_v(h, h->sq_val32);
    return square_tma_launch_v(h, h->sq_val);
}

template <bool UPDATE, bool EXACT, int SQ_U, bool HINTS, bool NOATOM = false>
void square_launch(cualign_bp *h)
{
    if (h->sq_val32) square_launch_v<UPDATE, EXACT, SQ_U, HINTS, NOATOM>(h, h->sq_val32);
    else square_launch_v<UPDATE, EXACT, SQ_U, HINTS, NOATOM>(h, h->sq_val);
}

cualign_status launch_square(cualign_bp *h, bool update, int64_t q0 = 0, int64_t q1 = -1)
{
    const bool exact = (h->flags & CUALIGN_FLAG_EXACT) != 0;
    if (update && !exact && (q0 != 0 || q1 >= 0)) {
        // a range of the squares (sharded: local-f / remote-f parts)
        KScope ks(h, CUALIGN_K_SQUARE);
        CA_TRY(square_tma_launch(h, q0, q1));
        CA_CUDA(cudaGetLastError());
        return CUALIGN_OK;
    }
    if (h->nsq > 0) {
        KScope ks(h, CUALIGN_K_SQUARE);
        if (update && exact) square_launch<true, true, 2, true>(h);
        else if (update) {
            static const int var = probe_knob("CUALIGN_SQ_VARIANT", 6); // probe build only (5, 8: timing probes)
            if (var == 6) CA_TRY(square_tma_launch(h));
            else if (var == 8) CA_TRY((square_tma_launch_v<double2, true>(h, h->sq_val))); // timing probe: no F sums
            else if (var == 0) square_launch<true, false, 1, false>(h);
            else if (var == 1) square_launch<true, false, 1, true>(h);
            else if (var == 2) square_launch<true, false, 2, false>(h);
            else if (var == 4) square_launch<true, false, 4, false>(h);
            else if (var == 5) square_launch<true, false, 2, true, true>(h); // timing probe only: no F sums
            else square_launch<true, false, 2, true>(h);
        } else if (exact) square_launch<false, true, 2, true>(h);
        else square_launch<false, false, 2, true>(h);
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

// gh[p] = (gamma^p, 1 - gamma^p) for p = 0..cap-1, computed on the host in
// fp64 exactly as the oracle does (reading Z2) and read by the kernels at
// gh[p_dev + 1], so an iteration can be replayed from a CUDA graph.
cualign_status ensure_gh(cualign_bp *h, int64_t pmax)
{
    if (pmax < h->gh_cap) return CUALIGN_OK;
    int64_t cap = h->gh_cap ? h->gh_cap : 1024; // doubles on demand (captured graphs are re-captured)
    while (cap <= pmax) cap *= 2;
    std::vector<double2> tab((size_t)cap);
    for (int64_t p = 0; p < cap; p++) {
        const double g = pow(h->gamma, (double)p);
        tab[(size_t)p] = make_double2(g, 1.0 - g);
    }
    double2 *nd = nullptr;
    CA_TRY(dalloc(h, &nd, (size_t)cap));
    CA_CUDA(cudaMemcpy(nd, tab.data(), sizeof(double2) * (size_t)cap, cudaMemcpyHostToDevice));
    if (h->gh_dev) {
        CA_CUDA(cudaStreamSynchronize(h->stream));
        dfree(h, h->gh_dev);
    }
    h->gh_dev = nd;
    h->gh_cap = cap;
    invalidate_graphs(h); // captured kernels hold the old table pointer
    return CUALIGN_OK;
}

namespace {

__global__ void k_iota_from(int64_t n, int64_t first, int32_t *__restrict__ x)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = (int32_t)(first + i);
}

// rowptr[v] = first k with key[k] >= v (key sorted ascending), v in [0, n]
__global__ void k_rowptr_from_sorted64(int64_t m, const int32_t *__restrict__ key, int64_t n,
                                       int64_t *__restrict__ rowptr)
{
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n;
         v += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = 0, hi = m;
        while (lo < hi) {
            const int64_t mid = lo + ((hi - lo) >> 1);
            if (key[mid] < (int32_t)v) lo = mid + 1;
            else hi = mid;
        }
        rowptr[v] = lo;
    }
}

__global__ void k_fill_neg_inf(int64_t n, double2 *__restrict__ x)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = make_double2(-INFINITY, -INFINITY);
}

// merge the world partial B-side top-2 arrays (gathered [world][nB]); max is
// exact, so the merged (max1, max2) equals the single-GPU one bit for bit
__global__ void k_merge_top2(int64_t nB, int world, const double2 *__restrict__ all, double2 *__restrict__ out)
{
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nB; b += (int64_t)gridDim.x * blockDim.x) {
        double m1 = -INFINITY, m2 = -INFINITY;
        for (int r = 0; r < world; r++) {
            const double2 o = all[(int64_t)r * nB + b];
            top2_merge(m1, m2, o.x, o.y);
        }
        out[b] = make_double2(m1, m2);
    }
}

__global__ void k_add_u64(int64_t n, unsigned long long *__restrict__ dst, const unsigned long long *__restrict__ src)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] += src[i];
}

} // namespace

cualign_status bp_merge_top2(cualign_bp *h)
{
    KScope ks(h, CUALIGN_K_TOP2);
    const int64_t nB = h->L.nB;
    if (nB) k_merge_top2<<<grid_for(nB, 256, h->num_sms * 8), 256, 0, h->stream>>>(nB, h->world, h->Btop_all, h->Btop);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status bp_add_u64(cualign_bp *h, unsigned long long *dst, const unsigned long long *src, int64_t n)
{
    KScope ks(h, CUALIGN_K_OTHER);
    if (n > 0) k_add_u64<<<grid_for(n, 256, h->num_sms * 8), 256, 0, h->stream>>>(n, dst, src);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

namespace {

// B incidence restricted to the owned edges [e0, e1) (ids ascending per b)
cualign_status build_local_incidence(cualign_bp *h)
{
    const int64_t nB = h->L.nB, ml = h->e1 - h->e0;
    CA_TRY(dalloc(h, &h->Bedge_loc, (size_t)(ml ? ml : 1)));
    CA_TRY(dalloc(h, &h->Bptr_loc, (size_t)nB + 1));
    TmpBuf kb, ib, tb_;
    CA_CUDA(tmalloc(h, kb, sizeof(int32_t) * (size_t)(ml ? ml : 1)));
    CA_CUDA(tmalloc(h, ib, sizeof(int32_t) * (size_t)(ml ? ml : 1)));
    int32_t *keys = (int32_t *)kb.p, *ids = (int32_t *)ib.p;
    void *tmp = nullptr;
    cualign_status st = CUALIGN_OK;
    if (ml) {
        k_iota_from<<<grid_for(ml, 256, h->num_sms * 8), 256, 0, h->stream>>>(ml, h->e0, ids);
        int end_bit = 1;
        while (end_bit < 31 && ((int64_t)1 << end_bit) < nB) end_bit++;
        size_t tb = 0;
        cub::DeviceRadixSort::SortPairs(nullptr, tb, h->L.Lb + h->e0, keys, ids, h->Bedge_loc, (int)ml, 0, end_bit,
                                        h->stream);
        if (tmalloc(h, tb_, tb ? tb : 1) != cudaSuccess) st = CUALIGN_ENOMEM;
        tmp = tb_.p;
        if (st == CUALIGN_OK)
            cub::DeviceRadixSort::SortPairs(tmp, tb, h->L.Lb + h->e0, keys, ids, h->Bedge_loc, (int)ml, 0, end_bit,
                                            h->stream);
    }
    if (st == CUALIGN_OK)
        k_rowptr_from_sorted64<<<grid_for(nB + 1, 256, h->num_sms * 8), 256, 0, h->stream>>>(ml, keys, nB,
                                                                                         h->Bptr_loc);
    CA_TRY(st);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

} // namespace

cualign_status bp_setup(cualign_bp *h)
{
    KScope ks(h, CUALIGN_K_INIT);
    const int64_t nA = h->L.nA, nB = h->L.nB;
    CA_TRY(dalloc(h, &h->Atop, (size_t)nA + 1));
    CA_TRY(dalloc(h, &h->Btop, (size_t)nB + 1));
    CA_TRY(dalloc(h, &h->Bcnt, (size_t)nB + 1));
    CA_CUDA(cudaMemsetAsync(h->Bcnt, 0, sizeof(unsigned int) * ((size_t)nB + 1), h->stream));
    if (!h->sq_ctr) {
        CA_TRY(dalloc(h, &h->sq_ctr, 2));
        CA_CUDA(cudaMemsetAsync(h->sq_ctr, 0, 2 * sizeof(unsigned int), h->stream));
    }
    const int64_t *Bptr = h->L.Bptr;
    if (h->world > 1) {
        // partial B-side top-2 over the owned edges, gathered and merged
        CA_TRY(build_local_incidence(h));
        Bptr = h->Bptr_loc;
        CA_TRY(dalloc(h, &h->Btop_part, (size_t)nB + 1));
        CA_TRY(dalloc(h, &h->Btop_all, (size_t)nB * h->world + 1));
        k_fill_neg_inf<<<grid_for(nB + 1, 256, h->num_sms * 8), 256, 0, h->stream>>>(nB + 1, h->Btop_part);
        CA_CUDA(cudaGetLastError());
    }
    // B-side chunks for k_top2
    CA_TRY(dalloc(h, &h->Bcp, (size_t)nB + 1));
    CA_CUDA(cudaMemsetAsync(h->Bcp, 0, sizeof(int64_t), h->stream));
    if (nB > 0) {
        TmpBuf cb, tb_;
        size_t tb = 0;
        CA_CUDA(tmalloc(h, cb, sizeof(int64_t) * (size_t)nB));
        int64_t *cnt = (int64_t *)cb.p;
        k_chunk_count<<<grid_for(nB, 256, h->num_sms * 8), 256, 0, h->stream>>>(nB, Bptr, cnt);
        CA_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, cnt, h->Bcp + 1, (int)nB, h->stream));
        CA_CUDA(tmalloc(h, tb_, tb ? tb : 1));
        CA_CUDA(cub::DeviceScan::InclusiveSum(tb_.p, tb, cnt, h->Bcp + 1, (int)nB, h->stream));
        CA_CUDA(cudaMemcpyAsync(&h->nchunks, h->Bcp + nB, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream));
    }
    CA_TRY(dalloc(h, &h->cdesc, (size_t)h->nchunks + 1));
    CA_TRY(dalloc(h, &h->Bct, (size_t)h->nchunks + 1));
    if (nB > 0)
        k_chunk_fill<<<grid_for(nB, 256, h->num_sms * 8), 256, 0, h->stream>>>(nB, h->Bcp, Bptr, h->cdesc);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status bp_fsum(cualign_bp *h)
{
    if (!(h->flags & CUALIGN_FLAG_EXACT))
        CA_CUDA(cudaMemsetAsync(h->tacc, 0, sizeof(unsigned long long) * (size_t)(h->L.m ? h->L.m : 1), h->stream));
    return launch_square(h, false);
}

// Start of an iteration: the device counter advances to this iteration p
// (kernels read gh[p]); per-vertex top-2 of y^p over the owned A rows and of
// z^p over the B columns (partial over the owned edges when sharded).
// per-vertex top-2 of the current y^p (A rows) and z^p (B columns)
cualign_status bp_top2(cualign_bp *h)
{
    if (h->L.m > 0) {
        KScope ks(h, CUALIGN_K_TOP2);
        const bool sh = h->world > 1;
        Top2Args T{(int64_t)(h->a1 - h->a0), h->nchunks, (int64_t)h->a0, h->L.Arow, h->cdesc, h->Bcp,
                   sh ? h->Bptr_loc : h->L.Bptr, sh ? h->Bedge_loc : h->L.Bedge, h->yp, h->zp, h->Atop,
                   sh ? h->Btop_part : h->Btop, h->Bct, h->Bcnt};
        // lanes per tile: CUALIGN_TOP2_TG (measurement knob), else the
        // capturing graph's choice (h->top2_tg), else TG_DEFAULT
        static const int tg_env = [] {
            const int x = probe_knob("CUALIGN_TOP2_TG", 0);
            return (x == 1 || x == 2 || x == 4 || x == 8) ? x : 0;
        }();
        const int tg = tg_env ? tg_env : (h->top2_tg ? h->top2_tg : TG_DEFAULT);
        // CUALIGN_TOP2_GRID (measurement knob): at most this many blocks per SM
        // (grid-stride tiles), leaving SM slots to a concurrent rounding
        static const int gcap_env = probe_knob("CUALIGN_TOP2_GRID", 0);
        const int gcap = gcap_env > 0 ? gcap_env * h->num_sms : (1 << 30);
        const int64_t nt = T.nA + T.nchunks;
        if (nt > 0) {
            if (tg == 1)
                CA_CUDA(launch_pdl(k_top2<1>, dim3(grid_for(nt, 256, gcap)), dim3(256), 0, h->stream, T));
            else if (tg == 2)
                CA_CUDA(launch_pdl(k_top2<2>, dim3(grid_for(nt * 2, 256, gcap)), dim3(256), 0, h->stream, T));
            else if (tg == 4)
                CA_CUDA(launch_pdl(k_top2<4>, dim3(grid_for(nt * 4, 256, gcap)), dim3(256), 0, h->stream, T));
            else
                CA_CUDA(launch_pdl(k_top2<8>, dim3(grid_for(nt * 8, 256, gcap)), dim3(256), 0, h->stream, T));
        }
        CA_CUDA(cudaGetLastError());
    }
    return CUALIGN_OK;
}

// Start of an iteration: the device counter advances to this iteration p.
// Unsharded, the top-2 inputs of iteration p were computed right after the
// k_edge of iteration p-1 (while y^p, z^p are still in L2 -- the square pass
// streams ~2 GB through it before the next iteration starts) or at init /
// set_state; sharded, the partial top-2 is computed here and then merged.
cualign_status bp_front_top2(cualign_bp *h)
{
    {
        KScope ks(h, CUALIGN_K_OTHER);
        CA_CUDA(launch_pdl(k_advance, dim3(1), dim3(1), 0, h->stream, h->p_dev));
    }
    if (h->world > 1) return bp_top2(h);
    return CUALIGN_OK;
}

// Lines 10-12 and 14-15 on the owned edges (k_edge).  y^c, z^c of iteration p
// are final after this, so the rounding of p may run concurrently with the
// square pass.
cualign_status bp_front_edge(cualign_bp *h)
{
    const bool exact = (h->flags & CUALIGN_FLAG_EXACT) != 0;
    const bool literal = (h->flags & CUALIGN_FLAG_OTHERMAX_LITERAL) != 0;
    const int64_t ml = h->e1 - h->e0;
    if (ml > 0) {
        KScope ks(h, CUALIGN_K_EDGE);
        EdgeArgs R{h->e0, h->e1, h->L.La, h->L.Lb, h->L.w, h->alpha, h->fp_inv, h->gh_dev, h->p_dev, h->tacc,
                   h->texact, h->Atop, h->Btop, h->yp, h->zp, h->yc, h->zc, h->d, h->u};
        constexpr int EPT = 2; // measured: EPT 2 (48 regs) 0.085 ms vs EPT 4 (66 regs) 0.098 ms on O
        const int grid = grid_for((ml + EPT - 1) / EPT, 256, 1 << 30);
        if (exact && literal) k_edge<EPT, true, true><<<grid, 256, 0, h->stream>>>(R);
        else if (exact) k_edge<EPT, true, false><<<grid, 256, 0, h->stream>>>(R);
        else if (literal) k_edge<EPT, false, true><<<grid, 256, 0, h->stream>>>(R);
        else {
            // measurement knob: 1 = 1 edge per thread, 4 = 4 edges per thread
            static const int var = probe_knob("CUALIGN_EDGE_VAR", 0);
            if (var == 1) k_edge<1, false, false><<<grid_for(ml, 256, 1 << 30), 256, 0, h->stream>>>(R);
            else if (var == 4) k_edge<4, false, false><<<grid_for((ml + 3) / 4, 256, 1 << 30), 256, 0, h->stream>>>(R);
            else CA_CUDA(launch_pdl(k_edge<EPT, false, false>, dim3(grid), dim3(256), 0, h->stream, R));
        }
        CA_CUDA(cudaGetLastError());
    }
    if (h->world == 1) CA_TRY(bp_top2(h)); // the next iteration's othermax inputs
    return CUALIGN_OK;
}

cualign_status bp_iterate_front(cualign_bp *h)
{
    CA_TRY(bp_front_top2(h));
    return bp_front_edge(h);
}

// Second half: lines 9, 13, 16 on the S values (the square pass).
cualign_status bp_iterate_back(cualign_bp *h)
{
    if (h->L.m > 0) CA_TRY(launch_square(h, true));
    return CUALIGN_OK;
}

// the square pass over squares [q0, q1) only (sharded overlap, shard.cu)
cualign_status bp_iterate_back_range(cualign_bp *h, int64_t q0, int64_t q1)
{
    if (h->L.m > 0 && q1 > q0) CA_TRY(launch_square(h, true, q0, q1));
    return CUALIGN_OK;
}

cualign_status bp_iterate(cualign_bp *h, int32_t n)
{
    if (!h->capturing) CA_TRY(ensure_gh(h, h->p + n));
    for (int32_t k = 0; k < n; k++) {
        CA_TRY(bp_iterate_front(h));
        CA_TRY(bp_iterate_back(h));
        h->p += 1;
    }
    return CUALIGN_OK;
}

namespace {
// every square {e < f} with e or f marked: (e, f, S^p_ef, S^p_fe), appended
// at an atomic cursor (order unspecified; at most cap written, all counted)
template <class V>
__global__ void k_sample_squares(int64_t nsq, const int2 *__restrict__ sq_ef, const V *__restrict__ sq_val,
                                 const unsigned char *__restrict__ mark, int64_t cap,
                                 unsigned long long *__restrict__ cnt, int2 *__restrict__ out_ef,
                                 double2 *__restrict__ out_v)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq;
         q += (int64_t)gridDim.x * blockDim.x) {
        const int2 ef = sq_ef[q];
        if (!(mark[ef.x] | mark[ef.y])) continue;
        const unsigned long long k = atomicAdd(cnt, 1ull);
        if ((int64_t)k < cap) {
            out_ef[k] = ef;
            out_v[k] = load_pair<false>(sq_val + q);
        }
    }
}
} // namespace

cualign_status bp_sample_squares(cualign_bp *h, const int32_t *edges, int64_t n, int64_t cap, int32_t *e_out,
                                 int32_t *f_out, double *v_ef, double *v_fe, int64_t *n_out)
{
    const int64_t m = h->L.m;
    std::vector<unsigned char> mk((size_t)(m ? m : 1), 0);
    for (int64_t i = 0; i < n; i++) {
        if (edges[i] < 0 || edges[i] >= m) {
            set_error("sample_squares: edge id %d outside [0, %lld)", edges[i], (long long)m);
            return CUALIGN_EINVAL;
        }
        mk[(size_t)edges[i]] = 1;
    }
    TmpBuf mb, cb, eb, vb;
    const int64_t c = cap > 0 ? cap : 0;
    CA_CUDA(tmalloc(h, mb, mk.size()));
    CA_CUDA(tmalloc(h, cb, sizeof(unsigned long long)));
    CA_CUDA(tmalloc(h, eb, sizeof(int2) * (size_t)(c ? c : 1)));
    CA_CUDA(tmalloc(h, vb, sizeof(double2) * (size_t)(c ? c : 1)));
    CA_CUDA(cudaMemcpyAsync(mb.p, mk.data(), mk.size(), cudaMemcpyHostToDevice, h->stream));
    CA_CUDA(cudaMemsetAsync(cb.p, 0, sizeof(unsigned long long), h->stream));
    if (h->nsq > 0) {
        KScope ks(h, CUALIGN_K_STATE);
        const int grid = grid_for(h->nsq, 256, h->num_sms * 8);
        if (h->sq_val32)
            k_sample_squares<<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_ef, h->sq_val32, (const unsigned char *)mb.p,
                                                          c, (unsigned long long *)cb.p, (int2 *)eb.p,
                                                          (double2 *)vb.p);
        else
            k_sample_squares<<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_ef, h->sq_val, (const unsigned char *)mb.p,
                                                          c, (unsigned long long *)cb.p, (int2 *)eb.p,
                                                          (double2 *)vb.p);
        CA_CUDA(cudaGetLastError());
    }
    unsigned long long total = 0;
    CA_CUDA(cudaMemcpyAsync(&total, cb.p, sizeof(total), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    const int64_t k = (int64_t)total < c ? (int64_t)total : c;
    if (k > 0) {
        std::vector<int2> ef((size_t)k);
        std::vector<double2> v((size_t)k);
        CA_CUDA(cudaMemcpy(ef.data(), eb.p, sizeof(int2) * (size_t)k, cudaMemcpyDeviceToHost));
        CA_CUDA(cudaMemcpy(v.data(), vb.p, sizeof(double2) * (size_t)k, cudaMemcpyDeviceToHost));
        for (int64_t i = 0; i < k; i++) {
            if (e_out) e_out[i] = ef[(size_t)i].x;
            if (f_out) f_out[i] = ef[(size_t)i].y;
            if (v_ef) v_ef[i] = v[(size_t)i].x;
            if (v_fe) v_fe[i] = v[(size_t)i].y;
        }
    }
    *n_out = (int64_t)total;
    return CUALIGN_OK;
}

cualign_status bp_scatter_Sp(cualign_bp *h, double *Sfull_dev)
{
    CA_TRY(ensure_sq_pos(h));
    KScope ks(h, CUALIGN_K_STATE);
    const int grid = grid_for(h->nsq, 256, h->num_sms * 8);
    if (h->nsq && h->sq_val32)
        k_scatter_Sp<<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_val32, h->sq_pos, Sfull_dev);
    else if (h->nsq)
        k_scatter_Sp<<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_val, h->sq_pos, Sfull_dev);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status bp_gather_Sp(cualign_bp *h, const double *Sfull_dev)
{
    CA_TRY(ensure_sq_pos(h));
    KScope ks(h, CUALIGN_K_STATE);
    const int grid = grid_for(h->nsq, 256, h->num_sms * 8);
    if (h->nsq && h->sq_val32)
        k_gather_Sp<<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_val32, h->sq_pos, Sfull_dev);
    else if (h->nsq)
        k_gather_Sp<<<grid, 256, 0, h->stream>>>(h->nsq, h->sq_val, h->sq_pos, Sfull_dev);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

} // namespace cualign
