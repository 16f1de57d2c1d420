// init.cu -- rows a1 (canonical L, incidences) and a2 (S construction, Alg. 3)
// of the hot path, plus input validation.
//
// S definition (§2): S_{(i,i'),(j,j')} = 1 iff (i,j) in E_A and
// (i',j') in E_B.  Alg. 3 loops, per L edge e = (i, i'),
// over the neighbours j of i and j' of i' and tests (j, j') in E_L.  Here the
// same set is enumerated from the other side: for each j in N_A(i), the L row
// of j (candidates (j, b), b ascending) is intersected with the sorted
// N_B(i') by binary search -- k*log(deg) instead of deg_B work per j, which
// bounds the cost at hub vertices.  One warp per edge e; the warp walks the
// concatenation of the L rows of e's A-neighbours 32 candidates at a time, so
// hits are emitted in ascending f with a ballot prefix (no sort).
// Two passes (count -> scan -> fill); the fill also writes the square layout
// (f > e suffix of each row), see DESIGN.md "Data layout".
#include "internal.cuh"

#include <cub/cub.cuh>
#include <math.h>

namespace cualign {

namespace {


#define FULL_MASK 0xffffffffu

// ---------------------------------------------------------------- validation
enum : int {
    E_ROWPTR = 1, E_COLRANGE = 2, E_SELFLOOP = 4, E_UNSORTED = 8, E_ASYM = 16,
    E_LRANGE = 32, E_LORDER = 64, E_WFINITE = 128
};

__device__ __forceinline__ bool bsearch_i32(const int32_t *x, int64_t lo, int64_t hi, int32_t v)
{
    while (lo < hi) {
        int64_t mid = lo + ((hi - lo) >> 1);
        int32_t xm = x[mid];
        if (xm < v) lo = mid + 1;
        else if (xm > v) hi = mid;
        else return true;
    }
    return false;
}

// One warp per row (hub rows of ~10^3 entries would serialise one thread):
// lanes take the row's entries; sortedness compares each entry with its left
// neighbour, symmetry binary-searches i in row c.
__global__ void k_check_graph(int32_t n, int64_t nnz, const int64_t *rp, const int32_t *col,
                              int *err)
{
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = warp; i < n; i += nwarps) {
        const int64_t lo = rp[i], hi = rp[i + 1];
        if (lo < 0 || hi < lo || hi > nnz) {
            if (lane == 0) atomicOr(err, E_ROWPTR);
            continue;
        }
        int bad = 0;
        for (int64_t x = lo + lane; x < hi; x += 32) {
            const int32_t c = col[x];
            if (c < 0 || c >= n) {
                bad |= E_COLRANGE;
                continue;
            }
            if (c == (int32_t)i) bad |= E_SELFLOOP;
            if (x > lo && c <= col[x - 1]) bad |= E_UNSORTED;
            const int64_t clo = rp[c], chi = rp[c + 1];
            if (clo < 0 || chi < clo || chi > nnz || !bsearch_i32(col, clo, chi, (int32_t)i)) bad |= E_ASYM;
        }
        bad = __reduce_or_sync(FULL_MASK, bad);
        if (lane == 0 && bad) atomicOr(err, bad);
    }
}

__global__ void k_check_edges(int64_t m, int32_t nA, int32_t nB, const int32_t *a,
                              const int32_t *b, const double *w, int *err)
{
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m;
         k += (int64_t)gridDim.x * blockDim.x) {
        int32_t ak = a[k], bk = b[k];
        if (ak < 0 || ak >= nA || bk < 0 || bk >= nB) atomicOr(err, E_LRANGE);
        if (w && !isfinite(w[k])) atomicOr(err, E_WFINITE);
        if (k + 1 < m) {
            int32_t an = a[k + 1], bn = b[k + 1];
            if (an < ak || (an == ak && bn <= bk)) atomicOr(err, E_LORDER);
        }
    }
}

// Arow[v] = first index k with key[k] >= v (key sorted ascending), v in [0, n]
__global__ void k_rowptr_from_sorted(int64_t m, const int32_t *key, int32_t n, int64_t *rowptr)
{
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n;
         v += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = 0, hi = m;
        while (lo < hi) {
            int64_t mid = lo + ((hi - lo) >> 1);
            if (key[mid] < (int32_t)v) lo = mid + 1;
            else hi = mid;
        }
        rowptr[v] = lo;
    }
}

__global__ void k_iota(int64_t m, int32_t *x)
{
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m;
         k += (int64_t)gridDim.x * blockDim.x)
        x[k] = (int32_t)k;
}

// -------------------------------------------------------------- S build
// One warp per L edge e = (i, i').  Candidates f are the L edges (j, b) with
// j in N_A(i) (rows of L, concatenated in ascending j => ascending f); f is a
// hit iff b in N_B(i').  Rows e in [e_begin, e_end); the count pass writes
// cnt[e] (global index), the fill pass reads row pointers relative to e_begin
// (a shard builds only its own rows).
// UPPER: only the squares {e < f} (f > e <=> j > i: no self loops), i.e. the
// A neighbours j > i -- half the candidates; the count pass writes ucnt only
// and the fill pass writes sq_ef only (the CSR is built on demand from the
// squares, see ensure_csr).
template <bool FILL, bool UPPER = false>
__global__ void __launch_bounds__(256)
k_sbuild(int64_t e_begin, int64_t e_end, const int32_t *__restrict__ La, const int32_t *__restrict__ Lb,
         const int64_t *__restrict__ Arow, const int64_t *__restrict__ Ap,
         const int32_t *__restrict__ Aj, const int64_t *__restrict__ Bp,
         const int32_t *__restrict__ Bj, int64_t *__restrict__ cnt, int64_t *__restrict__ ucnt,
         const int64_t *__restrict__ Srp, const int64_t *__restrict__ sq_rp,
         int32_t *__restrict__ Scol, int2 *__restrict__ sq_ef, const uint8_t *__restrict__ only = nullptr)
{
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const unsigned lt_mask = (1u << lane) - 1u;
    for (int64_t e = e_begin + warp; e < e_end; e += nwarps) {
        const int32_t i = La[e], ip = Lb[e];
        if (only && !only[i]) continue; // rows the group-map build leaves to this kernel
        const int64_t bs = Bp[ip], be = Bp[ip + 1];
        int64_t a_lo = Ap[i];
        const int64_t a_hi = Ap[i + 1];
        if (UPPER) { // first A neighbour j > i (rows sorted)
            int64_t lo = a_lo, hi = a_hi;
            while (lo < hi) {
                const int64_t mid = lo + ((hi - lo) >> 1);
                if (Aj[mid] <= i) lo = mid + 1;
                else hi = mid;
            }
            a_lo = lo;
        }
        int64_t total = 0, upper = 0, lower_cnt = 0, row0 = 0, sq0 = 0;
        if (FILL) {
            const int64_t r = e - e_begin;
            sq0 = sq_rp[r];
            if (!UPPER) {
                row0 = Srp[r];
                lower_cnt = (Srp[r + 1] - row0) - (sq_rp[r + 1] - sq0);
            }
        }
        if (be == bs) {
            if (!FILL && lane == 0) {
                if (!UPPER) cnt[e] = 0;
                ucnt[e] = 0;
            }
            continue;
        }
        for (int64_t xb = a_lo; xb < a_hi; xb += 32) {
            const int64_t x = xb + lane;
            int64_t lo = 0, len = 0;
            if (x < a_hi) {
                const int32_t j = Aj[x];
                lo = Arow[j];
                len = Arow[j + 1] - lo;
            }
            // inclusive warp scan of len
            int64_t incl = len;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                int64_t v = __shfl_up_sync(FULL_MASK, incl, off);
                if (lane >= off) incl += v;
            }
            const int64_t T = __shfl_sync(FULL_MASK, incl, 31);
            const int64_t excl = incl - len;
            for (int64_t c = 0; c < T; c += 32) {
                const int64_t pos = c + lane;
                // first lane k with incl[k] > pos
                int k = 0;
#pragma unroll
                for (int step = 16; step >= 1; step >>= 1) {
                    int64_t v = __shfl_sync(FULL_MASK, incl, k + step - 1);
                    if (v <= pos) k += step;
                }
                const int64_t ek = __shfl_sync(FULL_MASK, excl, k);
                const int64_t lk = __shfl_sync(FULL_MASK, lo, k);
                bool hit = false;
                int64_t f = 0;
                if (pos < T) {
                    f = lk + (pos - ek);
                    hit = bsearch_i32(Bj, bs, be, Lb[f]);
                }
                const unsigned mask = __ballot_sync(FULL_MASK, hit);
                if (FILL && UPPER) {
                    if (hit) sq_ef[sq0 + total + __popc(mask & lt_mask)] = make_int2((int)e, (int)f);
                } else if (FILL) {
                    if (hit) {
                        const int64_t idx = total + __popc(mask & lt_mask);
                        Scol[row0 + idx] = (int32_t)f;
                        if (idx >= lower_cnt) sq_ef[sq0 + (idx - lower_cnt)] = make_int2((int)e, (int)f);
                    }
                } else if (UPPER) {
                    // every candidate is an upper one
                } else {
                    const unsigned um = __ballot_sync(FULL_MASK, hit && f > e);
                    upper += __popc(um);
                }
                total += __popc(mask);
            }
        }
        if (!FILL && lane == 0) {
            if (!UPPER) cnt[e] = total;
            ucnt[e] = UPPER ? total : upper;
        }
    }
}

// Group-map S build of the squares {e < f} (unsharded init; DESIGN.md
// "S build").  One warp per A vertex i.  Every e = (i, i') of L's row i has
// the same candidates f = (j, j'), j in N_A(i), j > i (Alg. 3 :185-197, the
// upper half of row e), and (e, f) is a square iff j' in N_B(i').  The warp
// takes the edges of row i in groups of <= 32 whose B degrees sum to <= SBG_CAP
// and builds, in shared memory, the map j' -> {t : j' in N_B(b_t)} (a 32-bit
// lane mask) over the group; every candidate f is then ONE map lookup of its
// j', and each set bit t of the result is the square (e_t, f).  Per A vertex
// that is sum_t deg_B(b_t) inserts + (#candidates x #groups) lookups instead
// of one binary search per (e, f) pair.  An edge whose own B degree exceeds
// the map is a group of its own and tests its candidates by binary search in
// N_B(i') (the warp-per-e method).  Candidates run in ascending f, and an e
// gets at most one hit per f, so the hits of e arrive in ascending f: lane t
// keeps e_t's running count and the fill pass writes the same (e, f)-sorted
// layout as k_sbuild.  Counts are 32-bit scans: the caller checks n_B < 2^26.
constexpr int SBG_WARPS = 8;
constexpr int SBG_SLOTS = 512;   // hash slots per warp (key j', value lane mask)
constexpr int SBG_CAP = 256;     // inserts per group (load factor <= 1/2)
// candidates x row length above which a vertex's rows go to k_sbuild (warp
// per e): a bound on the lookups this one warp would make (one per candidate
// and group, at most one group per edge of the row)
constexpr int64_t SBG_HEAVY = (int64_t)1 << 22;

// 32 x 32 bit-matrix transpose across a warp: lane L holds row L (bit t =
// M[L][t]); afterwards lane t holds column t (bit L = M[L][t]).  Five
// butterfly steps swap the off-diagonal blocks of size 16, 8, 4, 2, 1.
__device__ __forceinline__ uint32_t warp_bit_transpose(uint32_t x, int lane)
{
    const uint32_t lowmask[5] = {0x0000ffffu, 0x00ff00ffu, 0x0f0f0f0fu, 0x33333333u, 0x55555555u};
#pragma unroll
    for (int s = 0; s < 5; s++) {
        const int j = 16 >> s;
        const uint32_t m = lowmask[s];
        const uint32_t y = __shfl_xor_sync(FULL_MASK, x, j);
        x = (lane & j) ? ((x & ~m) | ((y & ~m) >> j)) : ((x & m) | ((y & m) << j));
    }
    return x;
}

__device__ __forceinline__ int sbg_hash(int32_t b) { return (int)(((uint32_t)b * 2654435761u) >> 23); }

// first lane k whose inclusive sum exceeds pos (incl nondecreasing)
__device__ __forceinline__ int sbg_find(int32_t incl, int32_t pos)
{
    int k = 0;
#pragma unroll
    for (int step = 16; step >= 1; step >>= 1) {
        const int32_t v = __shfl_sync(FULL_MASK, incl, k + step - 1);
        if (v <= pos) k += step;
    }
    return k;
}

__device__ __forceinline__ int32_t sbg_scan(int32_t v, int lane)
{
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const int32_t o = __shfl_up_sync(FULL_MASK, v, off);
        if (lane >= off) v += o;
    }
    return v;
}

template <bool FILL>
__global__ void __launch_bounds__(SBG_WARPS * 32)
k_sbuild_g(int32_t nA, const int64_t *__restrict__ Arow, const int32_t *__restrict__ Lb,
           const int64_t *__restrict__ Ap, const int32_t *__restrict__ Aj, const int64_t *__restrict__ Bp,
           const int32_t *__restrict__ Bj, int64_t *__restrict__ ucnt, const int64_t *__restrict__ sq_rp,
           int2 *__restrict__ sq_ef, unsigned long long *__restrict__ next_i, uint8_t *__restrict__ heavy)
{
    __shared__ __align__(16) int32_t hkey_all[SBG_WARPS][SBG_SLOTS];
    __shared__ __align__(16) uint32_t hmask_all[SBG_WARPS][SBG_SLOTS];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    int32_t *hkey = hkey_all[wib];
    uint32_t *hmask = hmask_all[wib];
    const unsigned lt_mask = (1u << lane) - 1u;
    // dynamic A-vertex queue: a warp takes the next vertex when it finishes
    // one (hub vertices have up to ~10^4x the candidates of the median)
    while (true) {
        int64_t i = 0;
        if (lane == 0) i = (int64_t)atomicAdd(next_i, 1ull);
        i = __shfl_sync(FULL_MASK, i, 0);
        if (i >= nA) break;
        const int64_t l0 = Arow[i];
        const int ni = (int)(Arow[i + 1] - l0);
        if (ni == 0) continue;
        int64_t a_lo = Ap[i];
        const int64_t a_hi = Ap[i + 1];
        {
            int64_t lo = a_lo, hi = a_hi;
            while (lo < hi) {
                const int64_t mid = lo + ((hi - lo) >> 1);
                if (Aj[mid] <= (int32_t)i) lo = mid + 1;
                else hi = mid;
            }
            a_lo = lo;
        }
        if (a_lo == a_hi) continue; // no candidates: ucnt stays 0
        // heavy vertex (hub of A in R-MAT graphs): its candidates would be
        // walked once per group by this one warp; leave its rows to the
        // warp-per-e kernel
        // (one warp per L edge of the row).  The count pass decides, the
        // fill pass follows the flag.
        if (FILL) {
            if (heavy[i]) continue;
        } else {
            int64_t tot = 0;
            for (int64_t x = a_lo + lane; x < a_hi; x += 32) {
                const int32_t j = Aj[x];
                tot += Arow[j + 1] - Arow[j];
            }
#pragma unroll
            for (int off = 16; off >= 1; off >>= 1) tot += __shfl_xor_sync(FULL_MASK, tot, off);
            if (tot * ni > SBG_HEAVY) {
                if (lane == 0) {
                    heavy[i] = 1;
                    heavy[nA] = 1; // any heavy vertex: the warp-per-e passes run
                }
                continue;
            }
        }
        for (int t0 = 0; t0 < ni;) {
            // ---- next group: t0 .. t0+ng-1 with sum of B degrees <= SBG_CAP
            const int t = t0 + lane;
            int32_t bt = 0, bdeg = 0;
            if (t < ni) {
                bt = Lb[l0 + t];
                bdeg = (int32_t)(Bp[bt + 1] - Bp[bt]);
            }
            const int32_t dincl = sbg_scan(bdeg, lane);
            int ng = __popc(__ballot_sync(FULL_MASK, t < ni && dincl <= SBG_CAP));
            const bool single = ng == 0; // edge t0 alone exceeds the map
            if (single) ng = 1;
            const int64_t e_l = l0 + t;  // this lane's edge (valid for lane < ng)
            int64_t obase = 0;
            if (FILL && lane < ng) obase = sq_rp[e_l];
            int32_t cnt = 0;             // lane t: hits of e_{t0+t} so far
            if (!single) {
                // ---- build the map j' -> lanes over the group's B rows
                for (int q = lane; q < SBG_SLOTS / 4; q += 32) {
                    reinterpret_cast<int4 *>(hkey)[q] = make_int4(-1, -1, -1, -1);
                    reinterpret_cast<uint4 *>(hmask)[q] = make_uint4(0u, 0u, 0u, 0u);
                }
                __syncwarp();
                const int32_t gin = __shfl_sync(FULL_MASK, dincl, ng - 1);
                const int32_t dexcl = dincl - bdeg;
                const int64_t brow = (lane < ng) ? Bp[bt] : 0;
                for (int32_t c = 0; c < gin; c += 32) {
                    const int32_t pos = c + lane;
                    const int k = sbg_find(dincl, pos);
                    const int32_t ek = __shfl_sync(FULL_MASK, dexcl, k);
                    const int64_t rk = __shfl_sync(FULL_MASK, brow, k);
                    if (pos < gin) {
                        const int32_t jp = Bj[rk + (pos - ek)];
                        int slot = sbg_hash(jp);
                        while (true) {
                            const int32_t old = atomicCAS(&hkey[slot], -1, jp);
                            if (old == -1 || old == jp) break;
                            slot = (slot + 1) & (SBG_SLOTS - 1);
                        }
                        atomicOr(&hmask[slot], 1u << k);
                    }
                }
                __syncwarp();
            }
            const int32_t sb = __shfl_sync(FULL_MASK, bt, 0);
            const int64_t sblo = single ? Bp[sb] : 0, sbhi = single ? Bp[sb + 1] : 0;
            // ---- candidates f in ascending order: A neighbours j > i, L rows
            for (int64_t xb = a_lo; xb < a_hi; xb += 32) {
                const int64_t x = xb + lane;
                int64_t flo = 0;
                int32_t flen = 0;
                if (x < a_hi) {
                    const int32_t j = Aj[x];
                    flo = Arow[j];
                    flen = (int32_t)(Arow[j + 1] - flo);
                }
                const int32_t fincl = sbg_scan(flen, lane);
                const int32_t fT = __shfl_sync(FULL_MASK, fincl, 31);
                const int32_t fexcl = fincl - flen;
                for (int32_t c = 0; c < fT; c += 32) {
                    const int32_t pos = c + lane;
                    const int k = sbg_find(fincl, pos);
                    const int32_t ek = __shfl_sync(FULL_MASK, fexcl, k);
                    const int64_t lk = __shfl_sync(FULL_MASK, flo, k);
                    int64_t f = 0;
                    uint32_t hits = 0u;
                    if (pos < fT) {
                        f = lk + (pos - ek);
                        const int32_t jp = Lb[f];
                        if (single) {
                            hits = bsearch_i32(Bj, sblo, sbhi, jp) ? 1u : 0u;
                        } else {
                            int slot = sbg_hash(jp);
                            while (true) {
                                const int32_t key = hkey[slot];
                                if (key == jp) {
                                    hits = hmask[slot];
                                    break;
                                }
                                if (key < 0) break;
                                slot = (slot + 1) & (SBG_SLOTS - 1);
                            }
                        }
                    }
                    // lane t gets the lanes whose candidate hit e_t (bit transpose
                    // of the 32 hit masks): its count, and each hit's rank among
                    // the lower lanes = its place in row e_t (ascending f)
                    const uint32_t col = warp_bit_transpose(hits, lane);
                    if (FILL) {
                        const int R = __reduce_max_sync(FULL_MASK, (unsigned)__popc(hits));
                        uint32_t rem = hits;
                        for (int r = 0; r < R; r++) {
                            const bool has = rem != 0u;
                            const int tt = has ? __ffs(rem) - 1 : 0;
                            rem &= rem - 1u;
                            const uint32_t ct = __shfl_sync(FULL_MASK, col, tt);
                            const int32_t run = __shfl_sync(FULL_MASK, cnt, tt);
                            const int64_t ob = __shfl_sync(FULL_MASK, obase, tt);
                            if (has) sq_ef[ob + run + __popc(ct & lt_mask)] = make_int2((int)(l0 + t0 + tt), (int)f);
                        }
                    }
                    cnt += __popc(col);
                }
            }
            if (!FILL && lane < ng) ucnt[e_l] = cnt;
            __syncwarp();
            t0 += ng;
        }
    }
}

// lower-triangle row counts (row f gets one per square {e < f}); with the
// upper counts they give the full row lengths (max row -> fixed-point scale)
__global__ void k_lower_count(int64_t nsq, const int2 *__restrict__ sq_ef, unsigned int *__restrict__ lcnt)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq; q += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(lcnt + sq_ef[q].y, 1u);
}
__global__ void k_row_total(int64_t m, const int64_t *__restrict__ ucnt, const unsigned int *__restrict__ lcnt,
                            int64_t *__restrict__ cnt)
{
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x)
        cnt[e] = ucnt[e] + (int64_t)lcnt[e];
}
// CSR keys: (e, f) and (f, e) for every square {e < f}
__global__ void k_csr_keys(int64_t nsq, const int2 *__restrict__ sq_ef, unsigned long long *__restrict__ key)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq; q += (int64_t)gridDim.x * blockDim.x) {
        const int2 ef = sq_ef[q];
        key[q] = ((unsigned long long)(uint32_t)ef.x << 32) | (uint32_t)ef.y;
        key[nsq + q] = ((unsigned long long)(uint32_t)ef.y << 32) | (uint32_t)ef.x;
    }
}
__global__ void k_csr_cols(int64_t s, const unsigned long long *__restrict__ key, int32_t *__restrict__ col,
                           int32_t *__restrict__ row)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < s; q += (int64_t)gridDim.x * blockDim.x) {
        col[q] = (int32_t)(uint32_t)key[q];
        row[q] = (int32_t)(key[q] >> 32);
    }
}

// sq_pos[q] = (pos of (e,f) in row e, pos of (e) in row f): both by binary
// search in the sorted CSR rows, so it holds for any order of the squares
__device__ __forceinline__ int64_t lower_bound_i32(const int32_t *__restrict__ x, int64_t lo, int64_t hi, int32_t v)
{
    while (lo < hi) {
        const int64_t mid = lo + ((hi - lo) >> 1);
        if (x[mid] < v) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__global__ void k_sq_pos(int64_t nsq, const int2 *__restrict__ sq_ef, const int64_t *__restrict__ Srp,
                         const int32_t *__restrict__ Scol, longlong2 *__restrict__ sq_pos)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq;
         q += (int64_t)gridDim.x * blockDim.x) {
        const int2 ef = sq_ef[q];
        const int e = ef.x, f = ef.y;
        sq_pos[q] = make_longlong2(lower_bound_i32(Scol, Srp[e], Srp[e + 1], f),
                                   lower_bound_i32(Scol, Srp[f], Srp[f + 1], e));
    }
}

// Square tiles: the square pass gathers u[f] and
// adds into tacc[f] for the scattered endpoint f of every square.  Once m x 16 B
// exceeds L2 those become HBM sector misses, so the squares are ordered by
// (e block, f block) with blocks of 2^log_b edges -- inside a tile the
// scattered accesses stay in two blocks (2 x 2^log_b x 16 B, L2-resident) --
// and by (e, f) inside a tile (a stable sort of the (e, f)-sorted build).
__global__ void k_sq_tile_key(int64_t nsq, const int2 *__restrict__ sq_ef, int log_b, uint32_t nblocks,
                              uint32_t *__restrict__ key)
{
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nsq;
         q += (int64_t)gridDim.x * blockDim.x) {
        const int2 ef = sq_ef[q];
        key[q] = ((uint32_t)ef.x >> log_b) * nblocks + ((uint32_t)ef.y >> log_b);
    }
}

// ----------------------------------------------------------- partition
// Shard cost of an L edge: its squares (the square pass streams 40 B each)
// plus 2 (per-edge work ~ 80 B).  Boundaries at A-vertex row starts so every
// A row -- and with it othermaxrow -- stays on one shard.
__global__ void k_shard_cost(int64_t m, const int64_t *__restrict__ ucnt, int64_t *__restrict__ cost)
{
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x)
        cost[e] = ucnt[e] + 2;
}

// bnd[r] = first edge of shard r: the row start at or before the edge where
// the inclusive cost prefix first reaches total * r / P
__global__ void k_shard_bounds(int64_t m, const int64_t *__restrict__ prefix, const int32_t *__restrict__ La,
                               const int64_t *__restrict__ Arow, int P, int64_t *__restrict__ bnd)
{
    const int r = threadIdx.x;
    if (r > P) return;
    if (r == 0) {
        bnd[0] = 0;
        return;
    }
    if (r == P) {
        bnd[P] = m;
        return;
    }
    const double total = (double)prefix[m - 1];
    const int64_t target = (int64_t)(total * (double)r / (double)P);
    int64_t lo = 0, hi = m;
    while (lo < hi) {
        const int64_t mid = lo + ((hi - lo) >> 1);
        if (prefix[mid] < target) lo = mid + 1;
        else hi = mid;
    }
    bnd[r] = lo < m ? Arow[La[lo]] : m;
}

// undirected A edges as (i, j) pairs with i < j: the suffix of each sorted row
__global__ void k_upper_count(int64_t n, const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                              int64_t *__restrict__ cnt)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = rp[i], hi = rp[i + 1];
        const int64_t end = hi;
        while (lo < hi) { // first position with col > i
            const int64_t mid = lo + ((hi - lo) >> 1);
            if (col[mid] <= (int32_t)i) lo = mid + 1;
            else hi = mid;
        }
        cnt[i] = end - lo;
    }
}

// insert every undirected B edge {u < v} into the membership set
// one warp per B vertex (lanes over the row: hub rows do not serialise)
__global__ void k_bhash_insert(int64_t n, const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                               unsigned long long *__restrict__ T, int log2n)
{
    const uint64_t mask = (1ull << log2n) - 1;
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = warp; u < n; u += nwarps) {
        const int64_t hi = rp[u + 1];
        for (int64_t x = rp[u] + lane; x < hi; x += 32) {
            const int32_t v = col[x];
            if (v <= (int32_t)u) continue;
            const unsigned long long key = bhash_key((int32_t)u, v);
            for (uint64_t i = bhash_slot(key, log2n);; i = (i + 1) & mask) {
                const unsigned long long old = atomicCAS(T + i, BHASH_EMPTY, key);
                if (old == BHASH_EMPTY || old == key) break;
            }
        }
    }
}

__global__ void k_upper_fill(int64_t n, const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                             const int64_t *__restrict__ start, int2 *__restrict__ pairs)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t o = start[i];
        for (int64_t x = rp[i]; x < rp[i + 1]; x++)
            if (col[x] > (int32_t)i) pairs[o++] = make_int2((int)i, col[x]);
    }
}

cualign_status upload(cualign_bp *h, void **dst, const void *src, size_t bytes, bool device_ptrs)
{
    CA_TRY(dmalloc(h, dst, bytes));
    if (bytes)
        CA_CUDA(cudaMemcpyAsync(*dst, src, bytes,
                                device_ptrs ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                                h->stream));
    return CUALIGN_OK;
}

cualign_status check_flags(cualign_bp *h, int *err_dev, const char *what)
{
    int err = 0;
    CA_CUDA(cudaMemcpyAsync(&err, err_dev, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    if (err) {
        set_error("invalid %s:%s%s%s%s%s%s%s%s", what, (err & E_ROWPTR) ? " bad row pointers" : "",
                  (err & E_COLRANGE) ? " column out of range" : "",
                  (err & E_SELFLOOP) ? " self loop" : "",
                  (err & E_UNSORTED) ? " row not strictly increasing (unsorted/duplicate)" : "",
                  (err & E_ASYM) ? " not symmetric" : "",
                  (err & E_LRANGE) ? " edge endpoint out of range" : "",
                  (err & E_LORDER) ? " edges not strictly increasing in (a,b) (unsorted/duplicate)" : "",
                  (err & E_WFINITE) ? " non-finite weight" : "");
        return CUALIGN_EINVAL;
    }
    return CUALIGN_OK;
}

} // namespace

// ------------------------------------------------------------------ L build
cualign_status build_L(cualign_bp *h, LDev &L, const cualign_edges *E, bool device_ptrs,
                       bool validate, int32_t nA, int32_t nB)
{
    KScope ks(h, CUALIGN_K_INIT);
    // edge ids are int32 and the sorts below take an int count: reject an
    // oversized m before any upload or launch
    if (E->m >= ((int64_t)1 << 31) - 1) {
        set_error("m = %lld exceeds int32 edge ids", (long long)E->m);
        return CUALIGN_EINVAL;
    }
    L.nA = nA;
    L.nB = nB;
    L.m = E->m;
    const int64_t m = E->m;
    const int G = h->num_sms * 8;
    CA_TRY(upload(h, (void **)&L.La, E->a, sizeof(int32_t) * m, device_ptrs));
    CA_TRY(upload(h, (void **)&L.Lb, E->b, sizeof(int32_t) * m, device_ptrs));
    if (E->w) CA_TRY(upload(h, (void **)&L.w, E->w, sizeof(double) * m, device_ptrs));
    if (validate) {
        TmpBuf err;
        CA_CUDA(tmalloc(h, err, sizeof(int)));
        CA_CUDA(cudaMemsetAsync(err.p, 0, sizeof(int), h->stream));
        if (m) k_check_edges<<<grid_for(m, 256, G), 256, 0, h->stream>>>(m, nA, nB, L.La, L.Lb, L.w,
                                                                          (int *)err.p);
        CA_CUDA(cudaGetLastError());
        CA_TRY(check_flags(h, (int *)err.p, "L"));
    }
    // A-side rows: edges are sorted by a
    CA_TRY(dalloc(h, &L.Arow, (size_t)nA + 1));
    k_rowptr_from_sorted<<<grid_for((int64_t)nA + 1, 256, G), 256, 0, h->stream>>>(m, L.La, nA, L.Arow);
    CA_CUDA(cudaGetLastError());
    // B-side incidence: stable radix sort of edge ids by b (ids stay ascending)
    CA_TRY(dalloc(h, &L.Bedge, (size_t)(m ? m : 1)));
    CA_TRY(dalloc(h, &L.Bptr, (size_t)nB + 1));
    {
        TmpBuf keys_out, ids_in, tmp;
        CA_CUDA(tmalloc(h, keys_out, sizeof(int32_t) * (m ? m : 1)));
        CA_CUDA(tmalloc(h, ids_in, sizeof(int32_t) * (m ? m : 1)));
        if (m) {
            k_iota<<<grid_for(m, 256, G), 256, 0, h->stream>>>(m, (int32_t *)ids_in.p);
            int end_bit = 1;
            while (end_bit < 31 && ((int64_t)1 << end_bit) < (int64_t)nB) end_bit++;
            size_t tbytes = 0;
            CA_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tbytes, L.Lb, (int32_t *)keys_out.p,
                                                    (int32_t *)ids_in.p, L.Bedge, (int)m, 0, end_bit,
                                                    h->stream));
            CA_CUDA(tmalloc(h, tmp, tbytes ? tbytes : 1));
            CA_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tbytes, L.Lb, (int32_t *)keys_out.p,
                                                    (int32_t *)ids_in.p, L.Bedge, (int)m, 0, end_bit,
                                                    h->stream));
        }
        k_rowptr_from_sorted<<<grid_for((int64_t)nB + 1, 256, G), 256, 0, h->stream>>>(
            m, (int32_t *)keys_out.p, nB, L.Bptr);
        CA_CUDA(cudaGetLastError());
        CA_CUDA(cudaStreamSynchronize(h->stream)); // TmpBufs die here
    }
    return CUALIGN_OK;
}

// ------------------------------------------------------------ graph upload
cualign_status upload_graph(cualign_bp *h, const cualign_graph *g, const char *what, int64_t **rp, int32_t **col,
                            int64_t *nnz_out)
{
    const bool devp = (h->flags & CUALIGN_FLAG_DEVICE_PTRS) != 0;
    if (!g || g->n < 0 || !g->rowptr || (g->n > 0 && !g->col)) {
        set_error("invalid %s: NULL pointer or negative n", what);
        return CUALIGN_EINVAL;
    }
    // row pointers: read nnz (last entry) first
    int64_t nnz = 0;
    CA_CUDA(cudaMemcpy(&nnz, g->rowptr + g->n, sizeof(int64_t), devp ? cudaMemcpyDeviceToHost : cudaMemcpyHostToHost));
    if (nnz < 0 || nnz > ((int64_t)1 << 40)) {
        set_error("invalid %s: rowptr[n] out of range", what);
        return CUALIGN_EINVAL;
    }
    KScope ks(h, CUALIGN_K_INIT);
    CA_TRY(upload(h, (void **)rp, g->rowptr, sizeof(int64_t) * ((size_t)g->n + 1), devp));
    CA_TRY(upload(h, (void **)col, g->col, sizeof(int32_t) * (size_t)nnz, devp));
    TmpBuf err;
    CA_CUDA(tmalloc(h, err, sizeof(int)));
    CA_CUDA(cudaMemsetAsync(err.p, 0, sizeof(int), h->stream));
    if (g->n)
        k_check_graph<<<grid_for((int64_t)g->n * 32, 256, h->num_sms * 16), 256, 0, h->stream>>>(g->n, nnz, *rp, *col,
                                                                                   (int *)err.p);
    CA_CUDA(cudaGetLastError());
    CA_TRY(check_flags(h, (int *)err.p, what));
    *nnz_out = nnz;
    return CUALIGN_OK;
}

// ------------------------------------------------------------ problem build
// S for an unsharded handle: only the squares {e < f}
// are enumerated (half the candidates of the full rows), written straight
// into the square layout; nnz(S) = 2 x squares, and the full row lengths (for
// the fixed-point scale) come from a histogram of the squares' upper
// endpoints.  The CSR (get_S, exact mode, state transfer) is built from the
// squares only when one of those asks for it (ensure_csr).
static cualign_status build_S_upper(cualign_bp *h, const int64_t *Ap, const int32_t *Aj, const int64_t *Bp,
                                    const int32_t *Bj)
{
    const int64_t m = h->L.m;
    const int G = h->num_sms * 8;
    h->bounds.assign(2, 0);
    h->bounds[1] = m;
    h->e0 = 0;
    h->e1 = m;
    h->a0 = 0;
    h->a1 = h->L.nA;
    KScope ks(h, CUALIGN_K_INIT);
    TmpBuf ucnt, tmp, mx;
    CA_CUDA(tmalloc(h, ucnt, sizeof(int64_t) * (m ? m : 1)));
    CA_TRY(dalloc(h, &h->sq_rp, (size_t)m + 1));
    CA_CUDA(cudaMemsetAsync(h->sq_rp, 0, sizeof(int64_t), h->stream));
    h->nsq = 0;
    // group-map build (default) unless the 32-bit candidate counts could overflow
    static const int sb_env = probe_knob("CUALIGN_SBUILD_VAR", 1);
    const bool group_map = sb_env == 1 && h->L.nB < (1 << 26);
    const int32_t nA = h->L.nA;
    int sbg_blocks = 1;
    TmpBuf qctr, heavy;
    if (group_map) {
        // one resident wave; the warps pull A vertices from a queue
        int occ = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sbuild_g<true>, SBG_WARPS * 32, 0) != cudaSuccess ||
            occ < 1)
            occ = 1;
        (void)cudaGetLastError();
        sbg_blocks = grid_for((int64_t)nA * 32, SBG_WARPS * 32, (int64_t)occ * h->num_sms);
        CA_CUDA(tmalloc(h, qctr, 2 * sizeof(unsigned long long)));
        CA_CUDA(cudaMemsetAsync(qctr.p, 0, 2 * sizeof(unsigned long long), h->stream));
        CA_CUDA(tmalloc(h, heavy, (size_t)nA + 1));
        CA_CUDA(cudaMemsetAsync(heavy.p, 0, (size_t)nA + 1, h->stream));
    }
    const int old_blocks = grid_for(m * 32, 256, h->num_sms * 16);
    uint8_t any_heavy = 0;
    if (m) {
        if (group_map) {
            CA_CUDA(cudaMemsetAsync(ucnt.p, 0, sizeof(int64_t) * (size_t)m, h->stream));
            k_sbuild_g<false><<<sbg_blocks, SBG_WARPS * 32, 0, h->stream>>>(nA, h->L.Arow, h->L.Lb, Ap, Aj, Bp, Bj,
                                                                          (int64_t *)ucnt.p, nullptr, nullptr,
                                                                          (unsigned long long *)qctr.p,
                                                                          (uint8_t *)heavy.p);
            CA_CUDA(cudaMemcpyAsync(&any_heavy, (uint8_t *)heavy.p + nA, 1, cudaMemcpyDeviceToHost, h->stream));
            CA_CUDA(cudaStreamSynchronize(h->stream));
            if (any_heavy)
                k_sbuild<false, true><<<old_blocks, 256, 0, h->stream>>>(0, m, h->L.La, h->L.Lb, h->L.Arow, Ap, Aj,
                                                                         Bp, Bj, nullptr, (int64_t *)ucnt.p, nullptr,
                                                                         nullptr, nullptr, nullptr,
                                                                         (const uint8_t *)heavy.p);
        } else {
            const int blocks = grid_for(m * 32, 256, h->num_sms * 16);
            k_sbuild<false, true><<<blocks, 256, 0, h->stream>>>(0, m, h->L.La, h->L.Lb, h->L.Arow, Ap, Aj, Bp, Bj,
                                                                 nullptr, (int64_t *)ucnt.p, nullptr, nullptr,
                                                                 nullptr, nullptr);
        }
        CA_CUDA(cudaGetLastError());
        size_t tb = 0;
        CA_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, (int64_t *)ucnt.p, h->sq_rp + 1, (int)m, h->stream));
        CA_CUDA(tmalloc(h, tmp, tb ? tb : 1));
        CA_CUDA(cub::DeviceScan::InclusiveSum(tmp.p, tb, (int64_t *)ucnt.p, h->sq_rp + 1, (int)m, h->stream));
        CA_CUDA(cudaMemcpyAsync(&h->nsq, h->sq_rp + m, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream));
    }
    h->s = 2 * h->nsq;
    h->s_total = h->s;
    h->nsq_total = h->nsq;
    CA_TRY(dalloc(h, &h->sq_ef, (size_t)h->nsq + 2)); // +2: 16-byte bulk-copy tails
    const bool fp32 = (h->flags & CUALIGN_FLAG_FP32_S) != 0;
    if (fp32) CA_TRY(dalloc(h, &h->sq_val32, (size_t)h->nsq + 2));
    else CA_TRY(dalloc(h, &h->sq_val, (size_t)h->nsq + 2));
    h->max_row = 0;
    if (h->nsq) {
        if (group_map) {
            k_sbuild_g<true><<<sbg_blocks, SBG_WARPS * 32, 0, h->stream>>>(nA, h->L.Arow, h->L.Lb, Ap, Aj, Bp, Bj,
                                                                         nullptr, h->sq_rp, h->sq_ef,
                                                                         (unsigned long long *)qctr.p + 1,
                                                                         (uint8_t *)heavy.p);
            if (any_heavy)
                k_sbuild<true, true><<<old_blocks, 256, 0, h->stream>>>(0, m, h->L.La, h->L.Lb, h->L.Arow, Ap, Aj, Bp,
                                                                        Bj, nullptr, nullptr, nullptr, h->sq_rp,
                                                                        nullptr, h->sq_ef, (const uint8_t *)heavy.p);
        } else {
            const int blocks = grid_for(m * 32, 256, h->num_sms * 16);
            k_sbuild<true, true><<<blocks, 256, 0, h->stream>>>(0, m, h->L.La, h->L.Lb, h->L.Arow, Ap, Aj, Bp, Bj,
                                                                nullptr, nullptr, nullptr, h->sq_rp, nullptr,
                                                                h->sq_ef);
        }
        CA_CUDA(cudaGetLastError());
        // full row lengths: upper (ucnt) + lower (histogram of f) -> max row
        TmpBuf lcnt, tot, tmp2;
        CA_CUDA(tmalloc(h, lcnt, sizeof(unsigned int) * (size_t)m));
        CA_CUDA(tmalloc(h, tot, sizeof(int64_t) * (size_t)m));
        CA_CUDA(tmalloc(h, mx, sizeof(int64_t)));
        CA_CUDA(cudaMemsetAsync(lcnt.p, 0, sizeof(unsigned int) * (size_t)m, h->stream));
        k_lower_count<<<grid_for(h->nsq, 256, G), 256, 0, h->stream>>>(h->nsq, h->sq_ef, (unsigned int *)lcnt.p);
        k_row_total<<<grid_for(m, 256, G), 256, 0, h->stream>>>(m, (const int64_t *)ucnt.p,
                                                                (const unsigned int *)lcnt.p, (int64_t *)tot.p);
        CA_CUDA(cudaGetLastError());
        size_t tb = 0;
        CA_CUDA(cub::DeviceReduce::Max(nullptr, tb, (int64_t *)tot.p, (int64_t *)mx.p, (int)m, h->stream));
        CA_CUDA(tmalloc(h, tmp2, tb ? tb : 1));
        CA_CUDA(cub::DeviceReduce::Max(tmp2.p, tb, (int64_t *)tot.p, (int64_t *)mx.p, (int)m, h->stream));
        CA_CUDA(cudaMemcpyAsync(&h->max_row, mx.p, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
    }
    if (fp32) CA_CUDA(cudaMemsetAsync(h->sq_val32, 0, sizeof(float2) * ((size_t)h->nsq + 2), h->stream));
    else CA_CUDA(cudaMemsetAsync(h->sq_val, 0, sizeof(double2) * ((size_t)h->nsq + 2), h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    return CUALIGN_OK;
}

cualign_status build_problem(cualign_bp *h, const cualign_graph *A, const cualign_graph *B,
                             const cualign_edges *E)
{
    const bool devp = (h->flags & CUALIGN_FLAG_DEVICE_PTRS) != 0;
    const int G = h->num_sms * 8;
    int64_t nnzA = 0, nnzB = 0;
    int64_t *Ap = nullptr, *Bp = nullptr;
    int32_t *Aj = nullptr, *Bj = nullptr;
    CA_TRY(upload_graph(h, A, "graph A", &Ap, &Aj, &nnzA));
    CA_TRY(upload_graph(h, B, "graph B", &Bp, &Bj, &nnzB));
    init_trace(h, "upload graphs");
    CA_TRY(build_L(h, h->L, E, devp, true, A->n, B->n));
    init_trace(h, "build_L");
    const int64_t m = h->L.m;
    if (h->world == 1) {
        CA_TRY(build_S_upper(h, Ap, Aj, Bp, Bj));
    } else {
    // S: count pass over all rows (a shard needs every row's count for the
    // partition and the global max row), then this handle's rows [e0, e1)
    {
        KScope ks(h, CUALIGN_K_INIT);
        TmpBuf cnt, ucnt, tmp, mx, tot, bnd;
        CA_CUDA(tmalloc(h, cnt, sizeof(int64_t) * (m ? m : 1)));
        CA_CUDA(tmalloc(h, ucnt, sizeof(int64_t) * (m ? m : 1)));
        CA_CUDA(tmalloc(h, mx, 3 * sizeof(int64_t)));
        CA_CUDA(cudaMemsetAsync(mx.p, 0, 3 * sizeof(int64_t), h->stream));
        int64_t host3[3] = {0, 0, 0}; // max row, s, squares (global)
        if (m) {
            const int blocks = grid_for(m * 32, 256, h->num_sms * 16);
            k_sbuild<false><<<blocks, 256, 0, h->stream>>>(0, m, h->L.La, h->L.Lb, h->L.Arow, Ap, Aj, Bp, Bj,
                                                           (int64_t *)cnt.p, (int64_t *)ucnt.p, nullptr,
                                                           nullptr, nullptr, nullptr);
            CA_CUDA(cudaGetLastError());
            size_t t1 = 0, t3 = 0;
            CA_CUDA(cub::DeviceReduce::Max(nullptr, t3, (int64_t *)cnt.p, (int64_t *)mx.p, (int)m, h->stream));
            CA_CUDA(cub::DeviceReduce::Sum(nullptr, t1, (int64_t *)cnt.p, (int64_t *)mx.p + 1, (int)m, h->stream));
            size_t t2 = t1 > t3 ? t1 : t3;
            CA_CUDA(tmalloc(h, tmp, t2 ? t2 : 1));
            CA_CUDA(cub::DeviceReduce::Max(tmp.p, t3, (int64_t *)cnt.p, (int64_t *)mx.p, (int)m, h->stream));
            CA_CUDA(cub::DeviceReduce::Sum(tmp.p, t1, (int64_t *)cnt.p, (int64_t *)mx.p + 1, (int)m, h->stream));
            CA_CUDA(cub::DeviceReduce::Sum(tmp.p, t1, (int64_t *)ucnt.p, (int64_t *)mx.p + 2, (int)m, h->stream));
            CA_CUDA(cudaMemcpyAsync(host3, mx.p, sizeof(host3), cudaMemcpyDeviceToHost, h->stream));
        }
        CA_CUDA(cudaStreamSynchronize(h->stream));
        h->max_row = host3[0];
        h->s_total = host3[1];
        h->nsq_total = host3[2];
        if (h->s_total != 2 * h->nsq_total) {
            set_error("internal: S not symmetric (s=%lld, upper=%lld)", (long long)h->s_total,
                      (long long)h->nsq_total);
            return CUALIGN_ECUDA;
        }
        // partition (A-vertex blocks) -- identical on every shard
        h->bounds.assign((size_t)h->world + 1, 0);
        h->bounds[(size_t)h->world] = m;
        if (h->world > 1 && m) {
            CA_CUDA(tmalloc(h, tot, sizeof(int64_t) * (size_t)m));
            CA_CUDA(tmalloc(h, bnd, sizeof(int64_t) * ((size_t)h->world + 1)));
            k_shard_cost<<<grid_for(m, 256, G), 256, 0, h->stream>>>(m, (const int64_t *)ucnt.p, (int64_t *)tot.p);
            size_t tb = 0;
            TmpBuf tmp2;
            CA_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, (int64_t *)tot.p, (int64_t *)tot.p, (int)m, h->stream));
            CA_CUDA(tmalloc(h, tmp2, tb ? tb : 1));
            CA_CUDA(cub::DeviceScan::InclusiveSum(tmp2.p, tb, (int64_t *)tot.p, (int64_t *)tot.p, (int)m, h->stream));
            k_shard_bounds<<<1, 32, 0, h->stream>>>(m, (const int64_t *)tot.p, h->L.La, h->L.Arow, h->world,
                                                    (int64_t *)bnd.p);
            CA_CUDA(cudaGetLastError());
            CA_CUDA(cudaMemcpyAsync(h->bounds.data(), bnd.p, sizeof(int64_t) * ((size_t)h->world + 1),
                                    cudaMemcpyDeviceToHost, h->stream));
            CA_CUDA(cudaStreamSynchronize(h->stream));
        }
        h->e0 = h->bounds[(size_t)h->rank];
        h->e1 = h->bounds[(size_t)h->rank + 1];
        const int64_t ml = h->e1 - h->e0;
        h->a0 = 0;
        h->a1 = 0;
        if (h->world == 1) {
            h->a1 = A->n;
        } else if (ml > 0) {
            int32_t aa[2];
            CA_CUDA(cudaMemcpy(&aa[0], h->L.La + h->e0, sizeof(int32_t), cudaMemcpyDeviceToHost));
            CA_CUDA(cudaMemcpy(&aa[1], h->L.La + h->e1 - 1, sizeof(int32_t), cudaMemcpyDeviceToHost));
            h->a0 = aa[0];
            h->a1 = aa[1] + 1;
        }
        // local row pointers: scans over this shard's rows
        CA_TRY(dalloc(h, &h->Srp, (size_t)ml + 1));
        CA_TRY(dalloc(h, &h->sq_rp, (size_t)ml + 1));
        CA_CUDA(cudaMemsetAsync(h->Srp, 0, sizeof(int64_t), h->stream));
        CA_CUDA(cudaMemsetAsync(h->sq_rp, 0, sizeof(int64_t), h->stream));
        if (ml) {
            size_t tb = 0;
            TmpBuf tmp3;
            CA_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, (int64_t *)cnt.p + h->e0, h->Srp + 1, (int)ml,
                                                  h->stream));
            CA_CUDA(tmalloc(h, tmp3, tb ? tb : 1));
            CA_CUDA(cub::DeviceScan::InclusiveSum(tmp3.p, tb, (int64_t *)cnt.p + h->e0, h->Srp + 1, (int)ml,
                                                  h->stream));
            CA_CUDA(cub::DeviceScan::InclusiveSum(tmp3.p, tb, (int64_t *)ucnt.p + h->e0, h->sq_rp + 1, (int)ml,
                                                  h->stream));
            CA_CUDA(cudaMemcpyAsync(&h->s, h->Srp + ml, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
            CA_CUDA(cudaMemcpyAsync(&h->nsq, h->sq_rp + ml, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
            CA_CUDA(cudaStreamSynchronize(h->stream));
        } else {
            h->s = 0;
            h->nsq = 0;
        }
    }
    // S: fill pass over this handle's rows
    CA_TRY(dalloc(h, &h->Scol, (size_t)(h->s ? h->s : 1)));
    CA_TRY(dalloc(h, &h->sq_ef, (size_t)h->nsq + 2)); // +2: 16-byte bulk-copy tails
    const bool fp32 = (h->flags & CUALIGN_FLAG_FP32_S) != 0;
    if (fp32) CA_TRY(dalloc(h, &h->sq_val32, (size_t)h->nsq + 2));
    else CA_TRY(dalloc(h, &h->sq_val, (size_t)h->nsq + 2));
    {
        KScope ks(h, CUALIGN_K_INIT);
        if (h->e1 > h->e0 && h->s) {
            const int blocks = grid_for((h->e1 - h->e0) * 32, 256, h->num_sms * 16);
            k_sbuild<true><<<blocks, 256, 0, h->stream>>>(h->e0, h->e1, h->L.La, h->L.Lb, h->L.Arow, Ap, Aj, Bp,
                                                          Bj, nullptr, nullptr, h->Srp, h->sq_rp, h->Scol,
                                                          h->sq_ef);
            CA_CUDA(cudaGetLastError());
        }
        if (fp32) CA_CUDA(cudaMemsetAsync(h->sq_val32, 0, sizeof(float2) * ((size_t)h->nsq + 2), h->stream));
        else CA_CUDA(cudaMemsetAsync(h->sq_val, 0, sizeof(double2) * ((size_t)h->nsq + 2), h->stream));
    }
    }
    init_trace(h, "S build");
    CA_TRY(tile_squares(h));
    init_trace(h, "tile squares");
    // the graphs are not needed after S is built
    CA_CUDA(cudaStreamSynchronize(h->stream));
    // Evaluate counts overlapped edges by the definition: it
    // keeps B's CSR and the undirected A edges as a flat (i < j) pair list --
    // one pair per thread, no per-vertex imbalance at hubs.
    h->Bp = Bp;
    h->Bj = Bj;
    {
        KScope ks(h, CUALIGN_K_INIT);
        const int64_t nA = A->n;
        TmpBuf cntb, startb, tmpb;
        int64_t *cnt = nullptr, *start = nullptr;
        size_t tb = 0;
        h->nApairs = 0;
        if (nA > 0) {
            CA_CUDA(tmalloc(h, cntb, sizeof(int64_t) * (size_t)nA));
            CA_CUDA(tmalloc(h, startb, sizeof(int64_t) * (size_t)nA));
            cnt = (int64_t *)cntb.p;
            start = (int64_t *)startb.p;
            k_upper_count<<<grid_for(nA, 256, G), 256, 0, h->stream>>>(nA, Ap, Aj, cnt);
            CA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, start, (int)nA, h->stream));
            CA_CUDA(tmalloc(h, tmpb, tb ? tb : 1));
            CA_CUDA(cub::DeviceScan::ExclusiveSum(tmpb.p, tb, cnt, start, (int)nA, h->stream));
            int64_t last[2];
            CA_CUDA(cudaMemcpyAsync(&last[0], start + nA - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
            CA_CUDA(cudaMemcpyAsync(&last[1], cnt + nA - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
            CA_CUDA(cudaStreamSynchronize(h->stream));
            h->nApairs = last[0] + last[1];
        }
        cualign_status st = dalloc(h, &h->Apairs, (size_t)h->nApairs + 1);
        if (st == CUALIGN_OK && h->nApairs)
            k_upper_fill<<<grid_for(nA, 256, G), 256, 0, h->stream>>>(nA, Ap, Aj, start, h->Apairs);
        CA_TRY(st);
        CA_CUDA(cudaGetLastError());
        // E_B membership set for evaluate: >= 2 slots per undirected edge
        int lg = 4;
        while ((1ll << lg) < nnzB) lg++; // nnzB = 2 |E_B| directed entries
        h->Bhash_log = lg;
        CA_TRY(dalloc(h, &h->Bhash, (size_t)1 << lg));
        CA_CUDA(cudaMemsetAsync(h->Bhash, 0xff, sizeof(unsigned long long) << lg, h->stream));
        const int64_t nB = B->n;
        if (nB > 0)
            k_bhash_insert<<<grid_for(nB * 32, 256, h->num_sms * 16), 256, 0, h->stream>>>(nB, Bp, Bj, h->Bhash, lg);
        CA_CUDA(cudaGetLastError());
    }
    init_trace(h, "pairs + E_B set");
    dfree(h, Ap);
    dfree(h, Aj);
    // fixed-point scale for the F row sums: beta * max_row * 2^bits < 2^62
    {
        double bound = h->beta * (double)h->max_row;
        int bits = 52;
        if (bound > 0) {
            int ex = 0;
            frexp(bound, &ex); // bound < 2^ex
            bits = 61 - ex;
            if (bits > 1000) bits = 1000;
        }
        h->fp_bits = bits;
        h->fp_scale = ldexp(1.0, bits);
        h->fp_inv = ldexp(1.0, -bits);
    }
    return CUALIGN_OK;
}

// Reorder the squares into (e block, f block) tiles (see k_sq_tile_key).
// S^p is still all zero, so only (e, f) moves.  cualign_params.square_tile_log
// overrides the block size (-1 = keep the (e, f) order; result-neutral).
cualign_status tile_squares(cualign_bp *h)
{
    const int log_b = h->tile_log_param < 0 ? 0 : (h->tile_log_param > 0 ? h->tile_log_param : SQ_TILE_LOG);
    h->sq_tile_log = 0;
    if (log_b <= 0 || h->nsq < 2 || h->nsq >= INT32_MAX) return pack_squares(h);
    const uint32_t nblocks = (uint32_t)(((h->L.m - 1) >> log_b) + 1);
    if (nblocks < 2 || (uint64_t)nblocks * nblocks >= (1ull << 32)) return pack_squares(h);
    int end_bit = 1;
    while ((1ull << end_bit) < (uint64_t)nblocks * nblocks) end_bit++;
    const int n = (int)h->nsq;
    TmpBuf keys, keys2, tmp;
    int2 *sorted = nullptr;
    CA_CUDA(tmalloc(h, keys, sizeof(uint32_t) * (size_t)n));
    CA_CUDA(tmalloc(h, keys2, sizeof(uint32_t) * (size_t)n));
    CA_TRY(dalloc(h, &sorted, (size_t)n + 2));
    {
        KScope ks(h, CUALIGN_K_INIT);
        k_sq_tile_key<<<grid_for(n, 256, h->num_sms * 16), 256, 0, h->stream>>>(n, h->sq_ef, log_b, nblocks,
                                                                                (uint32_t *)keys.p);
        CA_CUDA(cudaGetLastError());
        size_t tb = 0;
        const unsigned long long *vin = reinterpret_cast<const unsigned long long *>(h->sq_ef);
        unsigned long long *vout = reinterpret_cast<unsigned long long *>(sorted);
        CA_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, (const uint32_t *)keys.p, (uint32_t *)keys2.p, vin,
                                                vout, n, 0, end_bit, h->stream));
        CA_CUDA(tmalloc(h, tmp, tb ? tb : 1));
        CA_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tb, (const uint32_t *)keys.p, (uint32_t *)keys2.p, vin, vout,
                                                n, 0, end_bit, h->stream));
        CA_CUDA(cudaMemsetAsync(sorted + n, 0, 2 * sizeof(int2), h->stream));
    }
    CA_CUDA(cudaStreamSynchronize(h->stream));
    dfree(h, h->sq_ef);
    h->sq_ef = sorted;
    h->sq_tile_log = log_b;
    return pack_squares(h);
}

// Packed square indices.  The squares
// are cut into chunks of <= SQP_CHUNK consecutive squares inside which every
// f lies in one 2^SQP_FBITS block (fb = its start) and every e in
// [eb, eb + 2^SQP_EBITS) with eb = the chunk's first e; square q then packs
// into one 32-bit word (e - eb) << SQP_FBITS | (f - fb), half of the int2.
// Windows of SQP_CHUNK squares are split by one warp each: "hard" cuts (window
// start, nsq_split, a new f block, e decreasing -- a new tile) come from
// ballots over the window, and inside each hard segment (e non-decreasing)
// the greedy e-range cuts are found by binary search on e from each chunk
// start.  Pass 1 counts the chunks per window, pass 2 writes descriptors and
// words.
constexpr int SQP_PACK_WARPS = 4;
template <bool FILL>
__global__ void __launch_bounds__(SQP_PACK_WARPS * 32)
k_sqp_pack(int64_t nsq, int64_t split, const int2 *__restrict__ sq_ef, int64_t *__restrict__ wcnt,
           int4 *__restrict__ desc, uint32_t *__restrict__ words)
{
    constexpr int NB = SQP_CHUNK / 32;
    constexpr int64_t ELIM = 1ll << SQP_EBITS;
    __shared__ int s_start[SQP_PACK_WARPS][SQP_CHUNK + 1];
    const int lane = threadIdx.x & 31;
    int *starts = s_start[threadIdx.x >> 5];
    const int64_t nwin = (nsq + SQP_CHUNK - 1) / SQP_CHUNK;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w < nwin; w += nwarps) {
        const int64_t q0 = w * SQP_CHUNK;
        const int len = (int)((q0 + SQP_CHUNK < nsq) ? SQP_CHUNK : nsq - q0);
        const int2 *__restrict__ W = sq_ef + q0;
        unsigned hm[NB];
#pragma unroll
        for (int k = 0; k < NB; k++) {
            const int r = lane + 32 * k;
            bool cut = false;
            if (r < len) {
                if (r == 0 || q0 + r == split) {
                    cut = true;
                } else {
                    const int2 ef = W[r], pv = W[r - 1];
                    cut = ((uint32_t)ef.y >> SQP_FBITS) != ((uint32_t)pv.y >> SQP_FBITS) || ef.x < pv.x;
                }
            }
            hm[k] = __ballot_sync(FULL_MASK, cut);
        }
        int nc = 0;
        if (lane == 0) {
            int r = 0;
            while (r < len) {
                // next hard cut after r
                int nh = len;
                for (int x = r + 1; x < len;) {
                    const unsigned m = hm[x >> 5] >> (x & 31);
                    if (m) {
                        nh = x + __ffs(m) - 1;
                        break;
                    }
                    x = (x | 31) + 1;
                }
                for (int c = r; c < nh;) {
                    starts[nc++] = c;
                    const int eb = W[c].x;
                    int lo = c + 1, hi = nh; // first index with e - eb >= ELIM
                    while (lo < hi) {
                        const int mid = (lo + hi) >> 1;
                        if ((int64_t)W[mid].x - eb >= ELIM) hi = mid;
                        else lo = mid + 1;
                    }
                    c = lo;
                }
                r = nh;
            }
            starts[nc] = len;
        }
        nc = __shfl_sync(FULL_MASK, nc, 0);
        __syncwarp();
        if (!FILL) {
            if (lane == 0) wcnt[w] = nc;
            __syncwarp();
            continue;
        }
        const int64_t cbase = w ? wcnt[w - 1] : 0; // wcnt: inclusive prefix after pass 1
        for (int c = lane; c < nc; c += 32) {
            const int2 e0 = W[starts[c]];
            desc[cbase + c] = make_int4((int)(q0 + starts[c]), starts[c + 1] - starts[c], e0.x,
                                        (int)(((uint32_t)e0.y >> SQP_FBITS) << SQP_FBITS));
        }
#pragma unroll 4
        for (int k = 0; k < NB; k++) {
            const int r = lane + 32 * k;
            if (r >= len) break;
            int lo = 0, hi = nc - 1; // chunk c with starts[c] <= r < starts[c + 1]
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (starts[mid] <= r) lo = mid;
                else hi = mid - 1;
            }
            const int2 e0 = W[starts[lo]], ef = W[r];
            const int fb = (int)(((uint32_t)e0.y >> SQP_FBITS) << SQP_FBITS);
            words[q0 + r] = ((uint32_t)(ef.x - e0.x) << SQP_FBITS) | (uint32_t)(ef.y - fb);
        }
        __syncwarp();
    }
}

// first chunk starting at or after q (chunk starts ascend)
__global__ void k_sqp_find(int64_t n, const int4 *__restrict__ desc, int64_t q, int64_t *__restrict__ out)
{
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (desc[mid].x < q) lo = mid + 1;
        else hi = mid;
    }
    *out = lo;
}

cualign_status pack_squares(cualign_bp *h)
{
    if (h->sqp_w) dfree(h, h->sqp_w);
    if (h->sqp_desc) dfree(h, h->sqp_desc);
    h->sqp_w = nullptr;
    h->sqp_desc = nullptr;
    h->sqp_nchunks = 0;
    h->sqp_split_chunk = 0;
    const int64_t n = h->nsq;
    if (n < 1 || n >= INT32_MAX) return CUALIGN_OK;
    const int64_t nwin = (n + SQP_CHUNK - 1) / SQP_CHUNK;
    TmpBuf cnt, tmp, res;
    CA_CUDA(tmalloc(h, cnt, sizeof(int64_t) * (size_t)nwin));
    CA_CUDA(tmalloc(h, res, sizeof(int64_t)));
    int64_t *wc = (int64_t *)cnt.p;
    KScope ks(h, CUALIGN_K_INIT);
    const int grid = grid_for(nwin * 32, SQP_PACK_WARPS * 32, h->num_sms * 16);
    k_sqp_pack<false><<<grid, SQP_PACK_WARPS * 32, 0, h->stream>>>(n, h->nsq_split, h->sq_ef, wc, nullptr, nullptr);
    CA_CUDA(cudaGetLastError());
    size_t tb = 0;
    CA_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, wc, wc, (int)nwin, h->stream));
    CA_CUDA(tmalloc(h, tmp, tb ? tb : 1));
    CA_CUDA(cub::DeviceScan::InclusiveSum(tmp.p, tb, wc, wc, (int)nwin, h->stream));
    int64_t nch = 0;
    CA_CUDA(cudaMemcpyAsync(&nch, wc + nwin - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    // chunks far below SQP_CHUNK (an untiled order over m > 2^SQP_FBITS
    // edges) would starve the bulk copies: keep the int2 stream then
    if (nch > 2 * nwin) return CUALIGN_OK;
    CA_TRY(dalloc(h, &h->sqp_w, (size_t)n + 8)); // +8: 16-byte bulk-copy tails
    CA_TRY(dalloc(h, &h->sqp_desc, (size_t)nch));
    CA_CUDA(cudaMemsetAsync(h->sqp_w + n, 0, 8 * sizeof(uint32_t), h->stream));
    k_sqp_pack<true><<<grid, SQP_PACK_WARPS * 32, 0, h->stream>>>(n, h->nsq_split, h->sq_ef, wc, h->sqp_desc, h->sqp_w);
    CA_CUDA(cudaGetLastError());
    int64_t sc = 0;
    if (h->nsq_split > 0) {
        k_sqp_find<<<1, 1, 0, h->stream>>>(nch, h->sqp_desc, h->nsq_split, (int64_t *)res.p);
        CA_CUDA(cudaGetLastError());
        CA_CUDA(cudaMemcpyAsync(&sc, res.p, sizeof(int64_t), cudaMemcpyDeviceToHost, h->stream));
    }
    CA_CUDA(cudaStreamSynchronize(h->stream));
    h->sqp_nchunks = nch;
    h->sqp_split_chunk = sc;
    return CUALIGN_OK;
}

// The CSR of S (Srp, Scol; rows ascending) from the squares: the keys
// (e, f) and (f, e) of every square {e < f}, radix-sorted, are exactly the
// CSR order.  Built on demand for an unsharded handle (get_S, exact mode,
// state transfer); a shard builds its rows' CSR at init.
cualign_status ensure_csr(cualign_bp *h)
{
    if (h->Scol || h->world > 1) return CUALIGN_OK;
    const int64_t m = h->L.m, s = h->s;
    CA_TRY(dalloc(h, &h->Srp, (size_t)m + 1));
    CA_TRY(dalloc(h, &h->Scol, (size_t)(s ? s : 1)));
    CA_CUDA(cudaMemsetAsync(h->Srp, 0, sizeof(int64_t) * ((size_t)m + 1), h->stream));
    if (s == 0) return CUALIGN_OK;
    if (s >= INT32_MAX) {
        set_error("CSR of S: nnz(S) = %lld too large for the on-demand build", (long long)s);
        return CUALIGN_ENOMEM;
    }
    KScope ks(h, CUALIGN_K_INIT);
    TmpBuf k1, k2, tmp, rows;
    CA_CUDA(tmalloc(h, k1, sizeof(unsigned long long) * (size_t)s));
    CA_CUDA(tmalloc(h, k2, sizeof(unsigned long long) * (size_t)s));
    CA_CUDA(tmalloc(h, rows, sizeof(int32_t) * (size_t)s));
    const int G = h->num_sms * 16;
    k_csr_keys<<<grid_for(h->nsq, 256, G), 256, 0, h->stream>>>(h->nsq, h->sq_ef, (unsigned long long *)k1.p);
    CA_CUDA(cudaGetLastError());
    int bits = 1;
    while ((1ll << bits) < m) bits++;
    size_t tb = 0;
    CA_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, tb, (const unsigned long long *)k1.p,
                                           (unsigned long long *)k2.p, (int)s, 0, 32 + bits, h->stream));
    CA_CUDA(tmalloc(h, tmp, tb ? tb : 1));
    CA_CUDA(cub::DeviceRadixSort::SortKeys(tmp.p, tb, (const unsigned long long *)k1.p, (unsigned long long *)k2.p,
                                           (int)s, 0, 32 + bits, h->stream));
    k_csr_cols<<<grid_for(s, 256, G), 256, 0, h->stream>>>(s, (const unsigned long long *)k2.p, h->Scol,
                                                          (int32_t *)rows.p);
    // row pointers: rowptr[e] = first position with row >= e
    k_rowptr_from_sorted<<<grid_for(m + 1, 256, G), 256, 0, h->stream>>>(s, (const int32_t *)rows.p, (int32_t)m,
                                                                          h->Srp);
    CA_CUDA(cudaGetLastError());
    CA_CUDA(cudaStreamSynchronize(h->stream));
    return CUALIGN_OK;
}

cualign_status ensure_sq_pos(cualign_bp *h)
{
    CA_TRY(ensure_csr(h));
    if (h->sq_pos || h->nsq == 0) return CUALIGN_OK;
    KScope ks(h, CUALIGN_K_INIT);
    CA_TRY(dalloc(h, &h->sq_pos, (size_t)h->nsq));
    k_sq_pos<<<grid_for(h->nsq, 256, h->num_sms * 16), 256, 0, h->stream>>>(h->nsq, h->sq_ef, h->Srp,
                                                                            h->Scol, h->sq_pos);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

} // namespace cualign
