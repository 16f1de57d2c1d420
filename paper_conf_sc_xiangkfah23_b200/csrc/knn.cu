// knn.cu -- NEXT-2: the kNN sparsification that builds L
// from given embeddings, Alg. 1 lines 7-14 (text :121):
// s(u, v) = cosine_similarity(Y_A(u), Y_B(v)) for all pairs, keep the k most
// similar B vertices of every A vertex (reading Z19).  The only dense
// contraction of the method, so it runs on the 5th-generation tensor cores:
//
//   k_knn_prep   unit rows (fp64 norm), rounded to bf16, written in the
//                128-byte-swizzled K-major tile image the MMA reads, so every
//                operand tile is ONE contiguous 1-D bulk copy (no tensor map)
//   k_knn_tc     per CTA: 128 A rows x a range of B column tiles.  Warp 0:
//                bulk-copy producer (A tile once, B tiles through an
//                NS-stage mbarrier ring).  Warp 1: TMEM allocation and the
//                single-thread tcgen05.mma issue (M=128, N=BN, K=16 per
//                instruction, bf16 in / fp32 accumulate) into one of two TMEM
//                accumulators.  Warps 2-9: epilogue, one A row per thread
//                of each TMEM lane quarter, two warps per quarter on
//                interleaved 32-column chunks; a chunk is tested against the
//                row's running k-th best by its max (FMNMX3 tree) first:
//                tcgen05.ld 32 columns at a time and a running top-k (values
//                above the row's current k-th best are inserted) -- the
//                n_A x n_B similarity matrix never leaves the SM.
//   k_knn_merge  per A row: merge the top-k of the column splits by
//                (similarity desc, B index asc), emit the row's k edges in
//                ascending B order (canonical L order).
//
// Precision: the products are of the bf16-rounded unit
// vectors with fp32 accumulation; oracle/knn.py computes the same similarity
// exactly, and the tests compare selections up to that accumulation error.
#include "internal.cuh"
#include "ptx.cuh"

#include <cuda_bf16.h>
#include <climits>
#include <math.h>

namespace cualign {

namespace {

using namespace ptx;

constexpr int KNN_BM = 128;       // A rows per CTA (MMA M)
constexpr int KNN_KMAX = 32;      // max neighbours per row
constexpr int KNN_CB = 16;        // per-row candidate buffer (entries above the row's k-th best)
// EH epilogue warps per TMEM lane quarter (column interleave), 2 when the
// per-row top-k arrays of both fit next to >= 2 B stages (k_knn_tc<BN, EH>)
template <int EH>
constexpr int knn_threads() { return (2 + 4 * EH) * 32; }

// Unit rows -> bf16 -> swizzled tile image.  Tile t holds rows [t*R, t*R+R),
// K-block kb (64 columns) of the tile at byte (t*KB + kb) * R*128, row rr at
// +rr*128, and the 16-byte chunk c of the row at position c ^ (rr % 8) (the
// Swizzle<3,4,3> pattern of SWIZZLE_128B).  Padding rows / columns are 0.
__global__ void k_knn_prep(const float *__restrict__ Y, int32_t n, int32_t d, int32_t KB, int32_t R,
                           int64_t rows_pad, __nv_bfloat16 *__restrict__ out, int *__restrict__ err)
{
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < rows_pad;
         r += (int64_t)gridDim.x * blockDim.x) {
        double inv = 0.0;
        if (r < n) {
            double ss = 0.0;
            for (int j = 0; j < d; j++) { // ascending coordinate order (as the oracle)
                const double y = (double)Y[r * d + j];
                ss = ss + y * y;
            }
            if (!isfinite(ss)) atomicOr(err, 1);
            if (ss > 0.0) inv = 1.0 / sqrt(ss);
        }
        const int64_t t = r / R, rr = r % R;
        for (int kb = 0; kb < KB; kb++) {
            __nv_bfloat16 *row = out + ((t * KB + kb) * (int64_t)R + rr) * 64;
            for (int c = 0; c < 8; c++) {
                __align__(16) __nv_bfloat16 v[8];
                for (int q = 0; q < 8; q++) {
                    const int j = kb * 64 + c * 8 + q;
                    double x = 0.0;
                    if (r < n && j < d && inv > 0.0) x = (double)Y[r * d + j] * inv;
                    v[q] = __double2bfloat16(x); // round to nearest even
                }
                *reinterpret_cast<uint4 *>(row + ((c ^ (int)(rr & 7)) * 8)) = *reinterpret_cast<const uint4 *>(v);
            }
        }
    }
}

// Partial top-k of one CTA: rows [rb*128, +128) x B tiles [t0, t1).
// Output pv / pi: [row][split][half][k] (unsorted), idx INT_MAX = empty.
template <int BN, int EH, int CPL>
__global__ void __launch_bounds__(knn_threads<EH>(), 1)
k_knn_tc(const uint8_t *__restrict__ Asw, const uint8_t *__restrict__ Bsw, int32_t n_a, int32_t n_b, int32_t KB,
         int32_t k, int32_t ntilesB, int32_t tiles_per_split, int32_t nstages, float *__restrict__ pv,
         int32_t *__restrict__ pi, int probe)
{
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // the swizzle atoms need 1024-byte aligned tiles: align the base explicitly
    uint8_t *smem = smem_raw + ((1024u - (smem_addr(smem_raw) & 1023u)) & 1023u);
    const uint32_t a_bytes = (uint32_t)KB * KNN_BM * 128;
    const uint32_t b_bytes = (uint32_t)KB * BN * 128;
    uint8_t *sA = smem;
    uint8_t *sB = smem + a_bytes;                         // nstages x b_bytes (multiples of 1024)
    float *tv_all = reinterpret_cast<float *>(sB + (size_t)nstages * b_bytes);          // [H][k][128]
    int32_t *ti_all = reinterpret_cast<int32_t *>(tv_all + EH * k * KNN_BM);  // [H][k][128]
    float *cv_all = reinterpret_cast<float *>(ti_all + EH * k * KNN_BM);      // [H][CB][128]
    int32_t *ci_all = reinterpret_cast<int32_t *>(cv_all + EH * KNN_CB * KNN_BM); // [H][CB][128]
    uint64_t *bars = reinterpret_cast<uint64_t *>(ci_all + EH * KNN_CB * KNN_BM);
    uint64_t *full = bars;                  // [nstages]
    uint64_t *empty = bars + nstages;       // [nstages]
    uint64_t *tfull = bars + 2 * nstages;   // [2]
    uint64_t *tempty = tfull + 2;           // [2]
    uint64_t *afull = tempty + 2;           // [1]
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(afull + 1);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int rb = blockIdx.x, split = blockIdx.y, nsplit = gridDim.y;
    const int t0 = split * tiles_per_split;
    const int t1 = min(ntilesB, t0 + tiles_per_split);
    const int ntiles = max(0, t1 - t0);

    if (threadIdx.x == 0) {
        for (int s = 0; s < nstages; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        for (int b = 0; b < 2; b++) {
            mbar_init(&tfull[b], 1);
            mbar_init(&tempty[b], 4 * EH);
        }
        mbar_init(afull, 1);
        fence_mbar_init();
    }
    if (warp == 1) tmem_alloc(tmem_slot, 2 * BN);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        // ---------------------------------------------------- producer
        if (lane == 0) {
            const uint64_t keep = policy_evict_last();   // B tiles are re-read by every row block
            const uint64_t once = policy_evict_first();
            mbar_expect_tx(afull, a_bytes);
            bulk_load(sA, Asw + (size_t)rb * a_bytes, a_bytes, afull, once);
            for (int i = 0; i < ntiles; i++) {
                const int s = i % nstages;
                if (i >= nstages) mbar_wait(&empty[s], (uint32_t)((i / nstages) - 1) & 1u);
                mbar_expect_tx(&full[s], b_bytes);
                bulk_load(sB + (size_t)s * b_bytes, Bsw + (size_t)(t0 + i) * b_bytes, b_bytes, &full[s], keep);
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------- MMA issuer
        if (lane == 0) {
            constexpr uint32_t idesc = idesc_bf16_f32(KNN_BM, BN);
            const uint32_t a_base = smem_addr(sA);
            mbar_wait(afull, 0);
            for (int i = 0; i < ntiles; i++) {
                const int s = i % nstages, buf = i & 1;
                mbar_wait(&full[s], (uint32_t)(i / nstages) & 1u);
                if (i >= 2) mbar_wait(&tempty[buf], (uint32_t)((i >> 1) - 1) & 1u);
                tc_fence_after();
                const uint32_t b_base = smem_addr(sB + (size_t)s * b_bytes);
                for (int kb = 0; kb < (probe == 2 ? 0 : KB); kb++) { // probe 2: no MMA (timing only)
#pragma unroll
                    for (int kk = 0; kk < 4; kk++) { // K = 16 bf16 = 32 bytes per instruction
                        const uint64_t ad = sw128_kmajor_desc(a_base + kb * (KNN_BM * 128) + kk * 32);
                        const uint64_t bd = sw128_kmajor_desc(b_base + kb * (BN * 128) + kk * 32);
                        mma_bf16(tmem + buf * BN, ad, bd, idesc, (kb | kk) ? 1u : 0u);
                    }
                }
                mma_commit(&empty[s]);   // smem stage free once these MMAs completed
                mma_commit(&tfull[buf]); // accumulator ready for the epilogue
            }
        }
    } else {
        // --------------------------------------------------- epilogue
        // warp w may read TMEM lanes 32*(w%4)..+31 only; the EH warps of
        // one quarter take interleaved 32-column chunks of each tile and keep
        // their own running top-k (merged by k_knn_merge)
        const int q = warp & 3;            // TMEM lane quarter this warp may access
        const int half = (warp - 2) >> 2;  // which chunks of a tile
        const int row = q * 32 + lane;     // A row within the block = TMEM lane
        float *tv = tv_all + half * k * KNN_BM;
        int32_t *ti = ti_all + half * k * KNN_BM;
        float *cv = cv_all + half * KNN_CB * KNN_BM;
        int32_t *ci = ci_all + half * KNN_CB * KNN_BM;
        for (int j = 0; j < k; j++) {
            tv[j * KNN_BM + row] = -INFINITY;
            ti[j * KNN_BM + row] = INT_MAX;
        }
        float thr = -INFINITY; // the row's k-th best (as of the last compaction)
        int thr_pos = 0, cnt = 0;
        // Entries above thr are appended to the row's candidate buffer (two
        // shared-memory stores); the buffer is folded into the top-k by the
        // whole warp at once when some lane could overflow it.  Folding takes
        // the buffered entries in column order with the same strict test as a
        // sequential scan, so the kept set (value desc, lowest index among
        // equals) is the sequential one; only the per-insertion rescan of the
        // k slots is batched instead of diverging the warp per element.
        auto fold = [&]() {
            for (int b = 0; b < cnt; b++) {
                const float val = cv[b * KNN_BM + row];
                if (!(val > thr)) continue;
                tv[thr_pos * KNN_BM + row] = val;
                ti[thr_pos * KNN_BM + row] = ci[b * KNN_BM + row];
                float wv = INFINITY;
                int wi = -1, wp = 0;
                for (int jj = 0; jj < k; jj++) { // new worst: lowest value, then highest index
                    const float x = tv[jj * KNN_BM + row];
                    const int xi = ti[jj * KNN_BM + row];
                    if (x < wv || (x == wv && xi > wi)) {
                        wv = x;
                        wi = xi;
                        wp = jj;
                    }
                }
                thr = wv;
                thr_pos = wp;
            }
            cnt = 0;
        };
        for (int i = 0; i < ntiles; i++) {
            const int buf = i & 1;
            mbar_wait(&tfull[buf], (uint32_t)(i >> 1) & 1u);
            tc_fence_after();
            const int vbase = (t0 + i) * BN;
            // CPL chunks of 32 columns per TMEM wait: their loads are issued
            // back to back, so the tcgen05.ld latency is paid once per CPL
            // chunks (the epilogue, not the MMA, bounds this kernel)
            const int nch = probe == 1 ? 0 : BN / 32; // probe 1: no epilogue (timing only)
#pragma unroll 1
            for (int c0 = half; c0 < nch; c0 += EH * CPL) {
                uint32_t r[CPL][32];
                __syncwarp(); // .sync.aligned load: reconverge after a fold
#pragma unroll
                for (int cc = 0; cc < CPL; cc++) {
                    const int c = c0 + cc * EH;
                    if (c < nch) tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * BN + c * 32), r[cc]);
                }
                tmem_ld_wait();
#pragma unroll
                for (int cc = 0; cc < CPL; cc++) {
                    const int c = c0 + cc * EH;
                    if (c >= nch) break;
                    const int v0 = vbase + c * 32;
                    if (v0 + 32 > n_b) { // padding columns of the last tile never enter
#pragma unroll
                        for (int j = 0; j < 32; j++)
                            if (v0 + j >= n_b) r[cc][j] = __float_as_uint(-INFINITY);
                    }
                    // chunk max first (FMNMX3 tree): after the first tiles almost
                    // every chunk of every row is below the row's k-th best
                    float m4[4];
#pragma unroll
                    for (int t = 0; t < 4; t++) {
                        float x = __uint_as_float(r[cc][8 * t]);
#pragma unroll
                        for (int j = 1; j < 8; j += 2)
                            x = fmaxf(fmaxf(x, __uint_as_float(r[cc][8 * t + j])),
                                      __uint_as_float(r[cc][8 * t + (j + 1 < 8 ? j + 1 : j)]));
                        m4[t] = x;
                    }
                    const bool pass = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3])) > thr;
                    if (!__any_sync(0xffffffffu, pass)) continue; // warp-uniform
#pragma unroll
                    for (int g = 0; g < 4; g++) {
                        // room for 8 more in every lane's buffer (warp-uniform fold)
                        if (__any_sync(0xffffffffu, cnt > KNN_CB - 8)) fold();
#pragma unroll
                        for (int jj = 0; jj < 8; jj++) {
                            const float val = __uint_as_float(r[cc][8 * g + jj]);
                            if (val > thr) {
                                cv[cnt * KNN_BM + row] = val;
                                ci[cnt * KNN_BM + row] = v0 + 8 * g + jj;
                                cnt++;
                            }
                        }
                    }
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tempty[buf]);
        }
        fold();
        const int64_t u = (int64_t)rb * KNN_BM + row;
        if (u < n_a) {
            const int64_t o = ((u * nsplit + split) * EH + half) * k;
            for (int j = 0; j < k; j++) {
                pv[o + j] = tv[j * KNN_BM + row];
                pi[o + j] = ti[j * KNN_BM + row];
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc(tmem, 2 * BN);
    }
}

// per A row: top-k of the splits' candidates by (value desc, index asc), then
// the k edges in ascending B order
__global__ void k_knn_merge(int32_t n_a, int32_t k, int32_t nsplit, const float *__restrict__ pv,
                            const int32_t *__restrict__ pi, int32_t *__restrict__ La, int32_t *__restrict__ Lb,
                            double *__restrict__ Lw)
{
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n_a; u += (int64_t)gridDim.x * blockDim.x) {
        float bv[KNN_KMAX];
        int bi[KNN_KMAX];
        for (int j = 0; j < k; j++) {
            bv[j] = -INFINITY;
            bi[j] = INT_MAX;
        }
        const int64_t base = u * (int64_t)nsplit * k;
        for (int64_t c = 0; c < (int64_t)nsplit * k; c++) {
            const float x = pv[base + c];
            const int xi = pi[base + c];
            if (xi == INT_MAX) continue;
            // worst kept: lowest value, then highest index
            int wp = 0;
            for (int j = 1; j < k; j++)
                if (bv[j] < bv[wp] || (bv[j] == bv[wp] && bi[j] > bi[wp])) wp = j;
            if (x > bv[wp] || (x == bv[wp] && xi < bi[wp])) {
                bv[wp] = x;
                bi[wp] = xi;
            }
        }
        // ascending B index (insertion sort, k <= 32)
        for (int j = 1; j < k; j++) {
            const float x = bv[j];
            const int xi = bi[j];
            int p = j - 1;
            while (p >= 0 && bi[p] > xi) {
                bv[p + 1] = bv[p];
                bi[p + 1] = bi[p];
                p--;
            }
            bv[p + 1] = x;
            bi[p + 1] = xi;
        }
        for (int j = 0; j < k; j++) {
            La[u * k + j] = (int32_t)u;
            Lb[u * k + j] = bi[j];
            Lw[u * k + j] = (double)bv[j];
        }
    }
}

template <int BN, int EH, int CPL = 1>
cualign_status knn_launch(cualign_bp *h, const uint8_t *Asw, const uint8_t *Bsw, int32_t n_a, int32_t n_b,
                          int32_t KB, int32_t k, float *pv, int32_t *pi, int32_t nsplit, int32_t tps,
                          int32_t nstages, size_t smem)
{
    auto fn = k_knn_tc<BN, EH, CPL>;
    CA_CUDA(cudaFuncSetAttribute((const void *)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int32_t ntilesB = (n_b + BN - 1) / BN;
    dim3 grid((unsigned)((n_a + KNN_BM - 1) / KNN_BM), (unsigned)nsplit);
    // CUALIGN_KNN_PROBE (timing probes, wrong results): 1 = no epilogue, 2 = no MMA
    static const int probe = probe_knob("CUALIGN_KNN_PROBE", 0); // probe build only
    fn<<<grid, knn_threads<EH>(), smem, h->stream>>>(Asw, Bsw, n_a, n_b, KB, k, ntilesB, tps, nstages, pv, pi,
                                                     probe);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

} // namespace

cualign_status knn_build(cualign_bp *h, const float *YA, int32_t n_a, const float *YB, int32_t n_b, int32_t d,
                         int32_t k, int32_t *La, int32_t *Lb, double *Lw)
{
    const bool devp = (h->flags & CUALIGN_FLAG_DEVICE_PTRS) != 0;
    const int32_t KB = (d + 63) / 64;
    // shared memory: A tile, B stages, per-row top-k arrays of EH epilogue
    // warps per TMEM lane quarter, barriers.  Two warps per quarter (the
    // epilogue is latency-bound with one warp per SMSP) when their arrays fit
    // next to >= 2 B stages of 128 columns; else one warp, BN = 256 for d <= 128
    const size_t a_bytes = (size_t)KB * KNN_BM * 128;
    int smem_optin = 0;
    {
        int dev = 0;
        CA_CUDA(cudaGetDevice(&dev));
        CA_CUDA(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    }
    auto fixed_for = [&](int eh) { return a_bytes + (size_t)eh * (k + KNN_CB) * KNN_BM * 8 + 256; };
    auto stages_for = [&](int eh, int bn) -> int32_t {
        const size_t f = fixed_for(eh) + 1024, bb = (size_t)KB * bn * 128;
        return f >= (size_t)smem_optin ? 0 : (int32_t)std::min<size_t>(4, ((size_t)smem_optin - f) / bb);
    };
    static const int eh_env = probe_knob("CUALIGN_KNN_EH", 1);
    const int EH = (eh_env >= 2 && stages_for(2, 128) >= 2) ? 2 : 1;
    const int BN = (EH == 1 && KB <= 2) ? 256 : 128;
    const int32_t nstages = stages_for(EH, BN);
    if (nstages < 1) {
        set_error("cualign_knn: d = %d needs more shared memory than available", d);
        return CUALIGN_EINVAL;
    }
    const size_t b_bytes = (size_t)KB * BN * 128;
    const size_t smem = fixed_for(EH) + (size_t)nstages * b_bytes + 1024; // +1024: alignment slack
    const int64_t rowsA = ((int64_t)n_a + KNN_BM - 1) / KNN_BM * KNN_BM;
    const int64_t rowsB = ((int64_t)n_b + BN - 1) / BN * BN;
    float *dA = nullptr, *dB = nullptr;
    __nv_bfloat16 *Asw = nullptr, *Bsw = nullptr;
    int *err = nullptr;
    const cudaMemcpyKind kind = devp ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    CA_TRY(dalloc(h, &dA, (size_t)n_a * d + 1));
    CA_TRY(dalloc(h, &dB, (size_t)n_b * d + 1));
    if (n_a) CA_CUDA(cudaMemcpyAsync(dA, YA, sizeof(float) * (size_t)n_a * d, kind, h->stream));
    if (n_b) CA_CUDA(cudaMemcpyAsync(dB, YB, sizeof(float) * (size_t)n_b * d, kind, h->stream));
    CA_TRY(dalloc(h, &Asw, (size_t)rowsA * KB * 64 + 64));
    CA_TRY(dalloc(h, &Bsw, (size_t)rowsB * KB * 64 + 64));
    CA_TRY(dalloc(h, &err, 1));
    CA_CUDA(cudaMemsetAsync(err, 0, sizeof(int), h->stream));
    const int G = h->num_sms * 8;
    {
        KScope ks(h, CUALIGN_K_INIT);
        if (rowsA) k_knn_prep<<<grid_for(rowsA, 128, G), 128, 0, h->stream>>>(dA, n_a, d, KB, KNN_BM, rowsA, Asw, err);
        if (rowsB) k_knn_prep<<<grid_for(rowsB, 128, G), 128, 0, h->stream>>>(dB, n_b, d, KB, BN, rowsB, Bsw, err);
        CA_CUDA(cudaGetLastError());
    }
    int e = 0;
    CA_CUDA(cudaMemcpyAsync(&e, err, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    if (e) {
        set_error("cualign_knn: non-finite embedding entries");
        return CUALIGN_EINVAL;
    }
    if (n_a == 0) return CUALIGN_OK;
    // column splits: enough CTAs for every SM, >= 4 B tiles per split (pipelining)
    const int32_t ntilesB = (int32_t)(rowsB / BN);
    const int32_t row_blocks = (int32_t)(rowsA / KNN_BM);
    int32_t nsplit = (2 * h->num_sms + row_blocks - 1) / row_blocks;
    nsplit = std::max(1, std::min(nsplit, std::max(1, ntilesB / 4)));
    const int32_t tps = (ntilesB + nsplit - 1) / nsplit;
    nsplit = (ntilesB + tps - 1) / tps;
    float *pv = nullptr;
    int32_t *pi = nullptr;
    CA_TRY(dalloc(h, &pv, (size_t)n_a * nsplit * EH * k));
    CA_TRY(dalloc(h, &pi, (size_t)n_a * nsplit * EH * k));
    int32_t *oa = La, *ob = Lb;
    double *ow = Lw;
    const int64_t m = (int64_t)n_a * k;
    if (!devp) {
        CA_TRY(dalloc(h, &oa, (size_t)m));
        CA_TRY(dalloc(h, &ob, (size_t)m));
        CA_TRY(dalloc(h, &ow, (size_t)m));
    }
    {
        KScope ks(h, CUALIGN_K_OTHER);
        const uint8_t *a8 = (const uint8_t *)Asw, *b8 = (const uint8_t *)Bsw;
        cualign_status lst;
        static const int cpl = probe_knob("CUALIGN_KNN_CPL", 1); // measured: CPL 1 / 2 / 4 = 4.15 / 4.44 / 6.41 ms at 65536^2
        if (BN == 256 && EH == 2) lst = knn_launch<256, 2>(h, a8, b8, n_a, n_b, KB, k, pv, pi, nsplit, tps, nstages, smem);
        else if (BN == 256 && cpl == 4) lst = knn_launch<256, 1, 4>(h, a8, b8, n_a, n_b, KB, k, pv, pi, nsplit, tps, nstages, smem);
        else if (BN == 256 && cpl == 2) lst = knn_launch<256, 1, 2>(h, a8, b8, n_a, n_b, KB, k, pv, pi, nsplit, tps, nstages, smem);
        else if (BN == 256) lst = knn_launch<256, 1>(h, a8, b8, n_a, n_b, KB, k, pv, pi, nsplit, tps, nstages, smem);
        else if (EH == 2) lst = knn_launch<128, 2>(h, a8, b8, n_a, n_b, KB, k, pv, pi, nsplit, tps, nstages, smem);
        else lst = knn_launch<128, 1>(h, a8, b8, n_a, n_b, KB, k, pv, pi, nsplit, tps, nstages, smem);
        CA_TRY(lst);
        k_knn_merge<<<grid_for(n_a, 128, G), 128, 0, h->stream>>>(n_a, k, nsplit * EH, pv, pi, oa, ob, ow);
        CA_CUDA(cudaGetLastError());
    }
    if (!devp) {
        CA_CUDA(cudaMemcpyAsync(La, oa, sizeof(int32_t) * (size_t)m, cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaMemcpyAsync(Lb, ob, sizeof(int32_t) * (size_t)m, cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaMemcpyAsync(Lw, ow, sizeof(double) * (size_t)m, cudaMemcpyDeviceToHost, h->stream));
    }
    CA_CUDA(cudaStreamSynchronize(h->stream));
    return CUALIGN_OK;
}

} // namespace cualign
