// match.cu -- rows a7 (rounding by 1/2-approximate matching) and a8
// (evaluate + best) of the hot path: Alg. 2 lines 17-24.
//
// The paper rounds with the locally-dominant algorithm (
// Preis [24], Halappanavar [10]).  Under a strict total order of the edges --
// (x desc, edge id asc), readings Z6/Z7 -- every locally-dominant schedule
// produces the same matching: the greedy one (pin P9).  Two schedules are
// implemented; both are bit-exact against the oracle's sort-greedy:
//
//  * SUITOR (default).  Every vertex of one side proposes to its heaviest
//    eligible neighbour whose current suitor is lighter; a CAS on the
//    neighbour's suitor slot (an edge id) installs the proposal and the
//    displaced suitor -- now owned by the same thread tile -- proposes again
//    (the Suitor algorithm of Manne & Halappanavar, a lock-free form of the
//    locally-dominant rule, here one-sided: see k_suitor).  One kernel, no
//    grid-wide barriers.  y^c and z^c are matched in the same launch.
//  * POINTER ROUNDS (CUALIGN_FLAG_MATCH_ROUNDS).  The paper's Phase 1 / Phase 2
//    as synchronous rounds in one persistent cooperative kernel: every vertex
//    points at its best eligible unmatched neighbour, mutual pointers match,
//    vertices whose target got matched re-point; grid.sync() between phases
//    replaces the Q_C / Q_N queues.  Kept for comparison (ablation).
//
// Evaluate (Eq. 1): weight(M) over the original w (Z9);
// overlap(M) counted straight from the paper's definition: the
// A edges {i, j} whose images (M(i), M(j)) are a B edge -- equal to x'Sx/2
// (pin P11), but it reads the 20 MB graph CSRs instead of scattered S rows;
// score = alpha*w + beta*overlap; M_y wins ties; best on a strict > (Z8).
#include "internal.cuh"

#include <climits>
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
    const double *x0, *x1;
    int32_t *candA, *candB; // POINTER ROUNDS: candidate pointers
    unsigned long long *suit; // SUITOR: suitor slots of the targets (packed, see suitor_key)
    int propose_from_b;     // SUITOR: proposing side
    int32_t *mates;         // [2 slots][2 instances][nA]; the round writes slot *wslot (RoundDev)
    const int *wslot;
    int32_t *mateA;         // device-side: mates + *wslot * 2 nA (set in the kernels)
    int32_t *mateB;         // [ninst][nB] (transient)
    int2 *mvA;              // (M_y(i), M_z(i)) as B vertices, for evaluate
    int *qcnt;              // Suitor rounds: sub-queue counters (reset by k_collect), or null
    RoundDev *rd;
    unsigned long long *work; // proposals (suitor) / rounds, spread counters
    unsigned long long *dbg;  // optional diagnostics (CUALIGN_MATCH_DEBUG)
    // DIST (sharded rounding, NEXT-1): the proposers are this shard's A rows
    // [p0, p0 + nPl) with edges [e0, e1); every target slot starts a round
    // from the global suitor (gx = fp64 bits of its weight, gi = its edge)
    int32_t p0, nPl, e0, e1;
    const unsigned long long *gx;
    const int32_t *gi;
    const int32_t *act; // active flag per (instance, local proposer)
    // deferred evaluate (pipelined graphs): exhausted proposers write nothing;
    // k_defer_fill presets this round's mate slot and mvA to -1 just before
    // k_collect, after the previous round's evaluate chose the slot
    int defer;
};

constexpr int WORK_SPREAD = 64, WORK_STRIDE = 16; // counter slots, 128 B apart
// evaluate blocks of 128 threads in every schedule (the weight sums' block
// partition must not depend on the schedule): small enough for a block to
// fit beside the 48-register square pass's 4 CTAs per SM
constexpr int NQ = 64;          // Suitor-round sub-queues (one atomic counter each, 32 B apart)
constexpr int QSTRIDE = 8;
constexpr int SUITOR_ROUNDS_MAXDEG = 64; // proposal rounds scan a proposer's row in one thread

__device__ __forceinline__ bool better(double xa, int ea, double xb, int eb)
{
    return eb < 0 || xa > xb || (xa == xb && ea < eb);
}

__device__ __forceinline__ const double *xk(const MatchParams &P, int k) { return k ? P.x1 : P.x0; }

// this round's mate slot (RoundDev: never the slot that holds bestM)
__device__ __forceinline__ int32_t *slot_mates(const MatchParams &P)
{
    return P.mates + (int64_t)(*(volatile const int *)P.wslot) * 2 * P.nA;
}

__device__ __forceinline__ void set_mv(int2 *mvA, int64_t a, int k, int b)
{
    int *p = reinterpret_cast<int *>(mvA + a);
    p[k] = b;
}

// ------------------------------------------------------------------ Suitor
// One-sided proposals.  In a bipartite graph whose preferences come from ONE
// global strict ranking of the edges (x desc, id asc), the stable matching is
// unique and equals the greedy matching; deferred acceptance from either side
// (each proposer repeatedly proposes to its best neighbour whose current
// suitor is worse, displacing it) reaches it in any order -- the Suitor
// algorithm restricted to one side.  The proposing side is the one with the
// smaller maximum degree (on the paper's workloads: the k candidates of each A
// vertex), so no tile ever scans a hub's list.
// Slot v in [0, ninst*nP): instance k, proposer r.  suitor[k*nT + t] = edge
// by which the current suitor proposes to target t (-1 = none).
// One G-lane tile per proposer: the lanes scan the proposer's list together
// (G x U edges per pass, the loads of a pass issued together), a tile argmax
// picks the heaviest eligible target, lane 0 attempts the CAS and the outcome
// is broadcast.
//
// Suitor slot (u64): 0 = empty, else (key(x) << 32) | e, key(x) = the bits of
// fp32(x) rounded toward -inf, plus 1 (x > 0 only, so the key is monotone
// non-decreasing in x and never 0).  Different keys order two proposals
// without loading the occupant's weight; equal keys (weights within an fp32
// ulp) fall back to the exact fp64 comparison, so the order is exactly
// (x desc, id asc).
__device__ __forceinline__ uint32_t suitor_key(double x)
{
    return __float_as_uint(__double2float_rd(x)) + 1u;
}

// does the proposal (xe, e) with key ke beat the occupant slot s of target t?
// The occupant's exact weight (needed only on equal keys) is x[es] for an
// edge of this process; in DIST mode an occupant from another shard can only
// be the round's initial global suitor, whose weight is gx[t].
template <bool DIST>
__device__ __forceinline__ bool beats(const MatchParams &P, const double *__restrict__ x, int k, int64_t nT, int t,
                                      double xe, int e, uint32_t ke, unsigned long long s)
{
    if (s == 0ull) return true;
    const uint32_t ks = (uint32_t)(s >> 32);
    if (ke != ks) return ke > ks;
    const int es = (int)(uint32_t)s;
    double xs;
    if (DIST && es == P.gi[k * nT + t]) xs = __longlong_as_double((long long)P.gx[k * nT + t]);
    else xs = __ldg(x + es);
    return better(xe, e, xs, es);
}

// The proposal chain of one tile: proposer `cur` of instance k proposes
// (filter0: starting with a filtered scan -- it lost a proposal or was
// displaced before), and every proposer it displaces continues in the same
// tile, until a proposal lands in a free slot or a proposer is exhausted.
template <int G, int U, bool DIST, class Tile>
__device__ __forceinline__ void suitor_chain(const MatchParams &P, Tile &tile, int lane, bool fromB, int64_t nP,
                                             int64_t nT, int k, int cur, bool filter0, int64_t wslot_id)
{
    const double *__restrict__ x = xk(P, k);
    unsigned long long *sT = P.suit + k * nT;
    const int64_t *__restrict__ rp = fromB ? P.Bptr : P.Arow;
    const int32_t *__restrict__ tgt = fromB ? P.La : P.Lb;   // target vertex of an edge
    const int32_t *__restrict__ own = fromB ? P.Lb : P.La;   // proposer vertex of an edge
    unsigned long long proposals = 0, scans = 0;
    // the first scan of a proposer skips the suitor filter (its best target
    // is tried directly; a better occupant sends it back to a filtered scan)
    bool filter = filter0;
    while (true) {
        scans++;
        // heaviest eligible neighbour of `cur` whose suitor is lighter; its
        // target and, on a filtered scan, the slot value seen (the CAS's
        // expected value; the unfiltered first scan reads the slot first --
        // an optimistic CAS on an unread slot serialises on popular targets)
        int best = -1, bt = -1;
        double bx = 0.0;
        unsigned long long bs = 0ull;
        const int hi = (int)rp[cur + 1]; // positions < m < 2^31: 32-bit index math
        for (int j0 = (int)rp[cur] + lane; j0 < hi; j0 += G * U) {
            int ee[U], tt[U];
            double xx[U];
            unsigned long long ss[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                const int j = j0 + u * G;
                ee[u] = -1;
                if (j < hi) {
                    const int e = fromB ? __ldg(P.Bedge + j) : j;
                    xx[u] = __ldg(x + e);
                    tt[u] = __ldg(tgt + e);
                    ee[u] = (xx[u] > 0.0) ? e : -1; // only x > 0 is eligible (Z6)
                }
            }
            if (filter) {
#pragma unroll
                for (int u = 0; u < U; u++) ss[u] = ee[u] >= 0 ? *(volatile unsigned long long *)(sT + tt[u]) : 0ull;
            }
#pragma unroll
            for (int u = 0; u < U; u++) {
                if (ee[u] < 0) continue;
                if (filter && !beats<DIST>(P, x, k, nT, tt[u], xx[u], ee[u], suitor_key(xx[u]), ss[u])) continue;
                if (better(xx[u], ee[u], bx, best)) {
                    best = ee[u];
                    bx = xx[u];
                    bt = tt[u];
                    bs = filter ? ss[u] : 0ull;
                }
            }
        }
        const bool filtered = filter;
        filter = true;
#pragma unroll
        for (int off = G / 2; off >= 1; off >>= 1) {
            const double ox = tile.shfl_xor(bx, off);
            const int oe = tile.shfl_xor(best, off);
            const int ot = tile.shfl_xor(bt, off);
            const unsigned long long os = tile.shfl_xor(bs, off);
            if (oe >= 0 && better(ox, oe, bx, best)) {
                bx = ox;
                best = oe;
                bt = ot;
                bs = os;
            }
        }
        if (best < 0) {      // tile-uniform after the all-reduce
            // exhausted: `cur` stays unmatched (nobody proposes to a
            // proposer), so this is its only mate write this round -- the
            // matched ones are written from the target slots by k_collect
            if (!DIST && lane == 0 && !P.defer) {
                if (fromB) {
                    P.mateB[k * nP + cur] = -1;
                } else {
                    slot_mates(P)[k * nP + cur] = -1;
                    set_mv(P.mvA, cur, k, -1);
                }
            }
            break;
        }
        int code = 0;        // 0 rescan, 1 done, 2 displaced
        int next = cur;
        if (lane == 0) {
            const int tb = bt;
            unsigned long long *slotp = sT + tb;
            const uint32_t kb = suitor_key(bx);
            const unsigned long long mine = ((unsigned long long)kb << 32) | (uint32_t)best;
            unsigned long long s = filtered ? bs : *(volatile unsigned long long *)slotp;
            // CAS loop: retry directly while our edge still beats the occupant,
            // rescan the list only when it does not
            while (beats<DIST>(P, x, k, nT, tb, bx, best, kb, s)) {
                const unsigned long long old = atomicCAS(slotp, s, mine);
                if (old == s) {
                    proposals++;
                    const int es = (int)(uint32_t)s;
                    if (s == 0ull || (DIST && (es < P.e0 || es >= P.e1))) {
                        code = 1; // free slot, or another shard's suitor (its owner re-proposes)
                    } else {
                        code = 2;
                        next = __ldg(own + es); // the displaced proposer proposes again
                    }
                    break;
                }
                s = old;
            }
        }
        code = tile.shfl(code, 0);
        if (code == 1) break;
        if (code == 2) cur = tile.shfl(next, 0);
    }
    // proposal counters spread over WORK_SPREAD slots (one global address
    // would serialise ~10^5 atomics in one L2 slice)
    if (lane == 0 && proposals) atomicAdd(P.work + (wslot_id % WORK_SPREAD) * WORK_STRIDE + k, proposals);
    if (P.dbg && lane == 0) {
        atomicMax(P.dbg + 0, scans);
        atomicAdd(P.dbg + 1, scans);
        if (scans > 8) atomicAdd(P.dbg + 2, 1ull);
        if (scans > 64) atomicAdd(P.dbg + 3, 1ull);
        atomicMax(P.dbg + 4, proposals);
    }
}

template <int G, int U, bool DIST, class Tile>
__device__ __forceinline__ void suitor_tile(const MatchParams &P, Tile &tile, int lane, bool fromB, int64_t nP,
                                            int64_t nT, int64_t slot)
{
    const int k = (int)(slot / nP);
    int cur = (int)(slot - k * nP);
    if (DIST) {
        if (!P.act[slot]) return; // settled (or exhausted) in an earlier round
        cur += P.p0;
    }
    suitor_chain<G, U, DIST>(P, tile, lane, fromB, nP, nT, k, cur, false, slot);
}

// ------------------------------------- Suitor in proposal rounds (A proposers)
// Round 0 (k_propose_round<FIRST>): every proposer's FIRST proposal, one
// thread per (instance, A row): the row (contiguous, ~k entries, L1-reused)
// is scanned for its best eligible edge and a CAS tries that target.
// Rounds 1..R: one thread per queued proposer -- those that lost a CAS to a
// better suitor and those a proposal displaced -- scanning its row for the
// best target whose CURRENT suitor it beats (filtered scan) and proposing.
// A thread never follows a displacement chain: the displaced proposer goes to
// the next round's queue, so every round is a flat pass with all its
// proposers in flight at once (no tile divergence, no chain tails).  Whatever
// is still queued after round R runs the chain form (k_suitor_q).  Any order
// of proposals reaches the same stable matching (= greedy, pin P9), so the
// schedule changes no result.  Config O, p = 80 (bulk-synchronous count):
// round 0 settles 87 % (M_y) / 61 % (M_z) of the proposers, 10 rounds settle
// all.  Queues: 3 buffers of NQ sub-queues (sub-queue = 32-entry chunk index
// mod NQ, one warp-aggregated atomic per chunk); round r reads buffer r % 3,
// writes (r + 1) % 3 and clears the counters of (r + 2) % 3, which round
// r + 1 writes (k_collect clears all of them for the next rounding).
constexpr int QBUF = 3;

__device__ __forceinline__ void queue_push(int push, int64_t chunk, int32_t *__restrict__ queue,
                                           int *__restrict__ qcnt, int64_t qcap)
{
    const unsigned mask = __ballot_sync(0xffffffffu, push >= 0);
    if (!mask) return;
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(mask) - 1;
    const int q = (int)(chunk % NQ);
    int base = 0;
    if (lane == leader) base = atomicAdd(qcnt + q * QSTRIDE, __popc(mask));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (push >= 0) queue[q * qcap + base + __popc(mask & ((1u << lane) - 1u))] = push;
}

// successful proposals (round info rounds_y / rounds_z): one atomic per
// warp and instance, spread over WORK_SPREAD counters
__device__ __forceinline__ void count_proposals(const MatchParams &P, bool proposed, int k, int64_t chunk)
{
    const unsigned b0 = __ballot_sync(0xffffffffu, proposed && k == 0);
    const unsigned b1 = __ballot_sync(0xffffffffu, proposed && k == 1);
    if ((threadIdx.x & 31) == 0) {
        unsigned long long *w = P.work + (chunk % WORK_SPREAD) * WORK_STRIDE;
        if (b0) atomicAdd(w, (unsigned long long)__popc(b0));
        if (b1) atomicAdd(w + 1, (unsigned long long)__popc(b1));
    }
}

// exclusive prefix of the NQ sub-queue counts into s_off[0..NQ] (one warp)
__device__ __forceinline__ void queue_offsets(const int *__restrict__ qcnt, int *s_off)
{
    if (threadIdx.x < 32) {
        const int c0 = qcnt[(2 * threadIdx.x) * QSTRIDE], c1 = qcnt[(2 * threadIdx.x + 1) * QSTRIDE];
        int v = c0 + c1;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const int o = __shfl_up_sync(0xffffffffu, v, off);
            if ((int)threadIdx.x >= off) v += o;
        }
        s_off[2 * threadIdx.x + 1] = v - c1;
        s_off[2 * threadIdx.x + 2] = v;
        if (threadIdx.x == 0) s_off[0] = 0;
    }
    __syncthreads();
}

__device__ __forceinline__ int queue_at(const int32_t *__restrict__ queue, const int *s_off, int64_t qcap, int idx)
{
    int lo = 0, hi = NQ; // sub-queue q with s_off[q] <= idx < s_off[q + 1]
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (s_off[mid] <= idx) lo = mid;
        else hi = mid;
    }
    return __ldg(queue + lo * qcap + (idx - s_off[lo]));
}

// One proposal of proposer `cur` of instance k (row scan, filtered unless
// FIRST, CAS); returns the proposer to queue for the next round (itself if it
// lost, the displaced one if it displaced a suitor) or -1.
template <int U, bool FIRST>
__device__ __forceinline__ int propose_once(const MatchParams &P, int64_t nP, int64_t nT, int k, int cur,
                                            bool &proposed)
{
    const double *__restrict__ x = xk(P, k);
    unsigned long long *sT = P.suit + k * nT;
    const int lo = (int)__ldg(P.Arow + cur), hi = (int)__ldg(P.Arow + cur + 1);
    int best = -1, bt = -1;
    double bx = 0.0;
    unsigned long long bs = 0ull;
    for (int j0 = lo; j0 < hi; j0 += U) {
        double xx[U];
        int tt[U];
        unsigned long long ss[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            if (j0 + u < hi) {
                xx[u] = __ldg(x + j0 + u);
                tt[u] = __ldg(P.Lb + j0 + u);
            }
        }
        if (!FIRST) {
#pragma unroll
            for (int u = 0; u < U; u++)
                ss[u] = (j0 + u < hi && xx[u] > 0.0) ? *(volatile unsigned long long *)(sT + tt[u]) : 0ull;
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const int j = j0 + u;
            if (j >= hi || !(xx[u] > 0.0)) continue; // only x > 0 is eligible (Z6)
            if (!FIRST && !beats<false>(P, x, k, nT, tt[u], xx[u], j, suitor_key(xx[u]), ss[u])) continue;
            if (better(xx[u], j, bx, best)) {
                best = j;
                bx = xx[u];
                bt = tt[u];
                bs = FIRST ? 0ull : ss[u];
            }
        }
    }
    if (best < 0) {
        if (!P.defer) {
            slot_mates(P)[k * nP + cur] = -1; // exhausted (see suitor_chain)
            set_mv(P.mvA, cur, k, -1);
        }
        return -1;
    }
    unsigned long long *sp = sT + bt;
    const uint32_t kb = suitor_key(bx);
    const unsigned long long mine = ((unsigned long long)kb << 32) | (uint32_t)best;
    unsigned long long s = FIRST ? *(volatile unsigned long long *)sp : bs;
    while (beats<false>(P, x, k, nT, bt, bx, best, kb, s)) {
        const unsigned long long old = atomicCAS(sp, s, mine);
        if (old == s) {
            proposed = true;
            return s ? (int)(k * nP + __ldg(P.La + (int)(uint32_t)s)) : -1; // the displaced one
        }
        s = old;
    }
    return (int)(k * nP + cur); // lost: next round
}

template <int U>
__global__ void __launch_bounds__(256) k_propose_first(MatchParams P, int32_t *__restrict__ qout,
                                                       int *__restrict__ cout, int64_t qcap)
{
    pdl_wait();
    const int64_t nP = P.nA, nT = P.nB;
    const int64_t slot = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int push = -1, k = 0;
    bool proposed = false;
    if (slot < P.ninst * nP) {
        k = (int)(slot / nP);
        push = propose_once<U, true>(P, nP, nT, k, (int)(slot - k * nP), proposed);
    }
    count_proposals(P, proposed, k, slot >> 5);
    queue_push(push, slot >> 5, qout, cout, qcap);
}

// Thread-level Suitor chains (no queues): the first proposal of every
// proposer, then the thread follows its chain -- the proposer it displaced,
// or itself after a lost CAS -- with filtered proposals until one lands in a
// free slot or a proposer is exhausted.
template <int U>
__global__ void __launch_bounds__(256) k_propose_chain(MatchParams P)
{
    pdl_wait();
    const int64_t nP = P.nA, nT = P.nB;
    const int64_t slot = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    bool proposed = false;
    int k = 0;
    unsigned long long nprop[2] = {0ull, 0ull};
    if (slot < P.ninst * nP) {
        k = (int)(slot / nP);
        int v = propose_once<U, true>(P, nP, nT, k, (int)(slot - k * nP), proposed);
        nprop[k] += proposed;
        while (v >= 0) {
            const int kk = (int)(v / nP);
            proposed = false;
            v = propose_once<U, false>(P, nP, nT, kk, (int)(v - kk * nP), proposed);
            nprop[kk] += proposed;
        }
    }
    for (int kk = 0; kk < 2; kk++) {
        unsigned long long c = nprop[kk];
#pragma unroll
        for (int off = 16; off >= 1; off >>= 1) c += __shfl_down_sync(0xffffffffu, c, off);
        if ((threadIdx.x & 31) == 0 && c) atomicAdd(P.work + ((slot >> 5) % WORK_SPREAD) * WORK_STRIDE + kk, c);
    }
}

template <int U>
__global__ void __launch_bounds__(256) k_propose_round(MatchParams P, const int32_t *__restrict__ qin,
                                                       const int *__restrict__ cin, int32_t *__restrict__ qout,
                                                       int *__restrict__ cout, int *__restrict__ cclr, int64_t qcap)
{
    __shared__ int s_off[NQ + 1];
    pdl_wait();
    if (blockIdx.x == 0 && threadIdx.x < NQ) cclr[threadIdx.x * QSTRIDE] = 0;
    queue_offsets(cin, s_off);
    const int total = s_off[NQ];
    const int64_t nP = P.nA, nT = P.nB;
    const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = gwarp * 32; base < total; base += nwarps * 32) {
        const int idx = (int)(base + (threadIdx.x & 31));
        int push = -1, k = 0;
        bool proposed = false;
        if (idx < total) {
            const int v = queue_at(qin, s_off, qcap, idx);
            k = (int)(v / nP);
            push = propose_once<U, false>(P, nP, nT, k, (int)(v - k * nP), proposed);
        }
        count_proposals(P, proposed, k, base >> 5);
        queue_push(push, base >> 5, qout, cout, qcap);
    }
}

// After the last round: one wave of G-lane tiles over what is still queued,
// each running the Suitor chain (displaced proposers continue in the tile)
// until the matching is complete.
template <int G, int U, int MINB>
__global__ void __launch_bounds__(128, MINB) k_suitor_q(MatchParams P, const int32_t *__restrict__ queue,
                                                        const int *__restrict__ qcnt, int64_t qcap)
{
    __shared__ int s_off[NQ + 1];
    pdl_wait();
    queue_offsets(qcnt, s_off);
    auto tile = cg::tiled_partition<G>(cg::this_thread_block());
    const int lane = tile.thread_rank();
    const int64_t nP = P.nA, nT = P.nB;
    const int total = s_off[NQ];
    const int T = (int)(((int64_t)gridDim.x * blockDim.x) / G);
    for (int idx = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / G); idx < total; idx += T) {
        const int v = queue_at(queue, s_off, qcap, idx);
        const int k = (int)(v / nP);
        suitor_chain<G, U, false>(P, tile, lane, false, nP, nT, k, (int)(v - k * nP), true, idx);
    }
}

template <int G, int U, bool DIST = false, int MINB = 1>
__global__ void __launch_bounds__(128, MINB) k_suitor(MatchParams P)
{
    pdl_wait();
    auto tile = cg::tiled_partition<G>(cg::this_thread_block());
    const int lane = tile.thread_rank();
    const bool fromB = !DIST && P.propose_from_b != 0;
    const int64_t nP = DIST ? P.nPl : (fromB ? P.nB : P.nA);
    const int64_t nT = fromB ? P.nA : P.nB;
    const int64_t slot = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / G;
    if (slot < P.ninst * nP) suitor_tile<G, U, DIST>(P, tile, lane, fromB, nP, nT, slot);
}

// Persistent form: one wave of tiles, tile t proposes for slots t, t + T,
// t + 2T, ... -- a tile whose proposer runs a long displacement chain delays
// only its own later slots, instead of holding its whole block (and the
// block's SM slot) until its last tile finishes.
template <int G, int U, int MINB>
__global__ void __launch_bounds__(128, MINB) k_suitor_persistent(MatchParams P)
{
    auto tile = cg::tiled_partition<G>(cg::this_thread_block());
    const int lane = tile.thread_rank();
    const bool fromB = P.propose_from_b != 0;
    const int64_t nP = fromB ? P.nB : P.nA;
    const int64_t nT = fromB ? P.nA : P.nB;
    const int64_t T = ((int64_t)gridDim.x * blockDim.x) / G;
    for (int64_t slot = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / G; slot < P.ninst * nP; slot += T)
        suitor_tile<G, U, false>(P, tile, lane, fromB, nP, nT, slot);
}

// ------------------------------------------------- DIST round helper kernels
// slots of a round start from the global suitors
__global__ void k_dist_init_slots(int64_t n, const unsigned long long *__restrict__ gx, const int32_t *__restrict__ gi,
                                  unsigned long long *__restrict__ sT)
{
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int e = gi[v];
        sT[v] = e < 0 ? 0ull
                      : ((unsigned long long)suitor_key(__longlong_as_double((long long)gx[v])) << 32) | (uint32_t)e;
    }
}

// local winner per target -> (weight bits, edge) for the global merge; x > 0
// for every suitor, so the fp64 bits order like the weights
__global__ void k_dist_pack(int64_t nB, const unsigned long long *__restrict__ sT, const unsigned long long *__restrict__ gx,
                            const int32_t *__restrict__ gi, const double *__restrict__ x0, const double *__restrict__ x1,
                            unsigned long long *__restrict__ wxl, unsigned long long *__restrict__ wxg,
                            int32_t *__restrict__ wid)
{
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < 2 * nB; v += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long s = sT[v];
        unsigned long long bits = 0ull;
        int32_t e = INT_MAX;
        if (s) {
            e = (int32_t)(uint32_t)s;
            bits = (e == gi[v]) ? gx[v] : (unsigned long long)__double_as_longlong((v < nB ? x0 : x1)[e]);
        }
        wxl[v] = bits;
        wxg[v] = bits;
        wid[v] = e;
    }
}

// among the shards whose winner has the global max weight, the lowest edge id wins (Z7)
__global__ void k_dist_cand(int64_t n, const unsigned long long *__restrict__ wxl, const unsigned long long *__restrict__ wxg,
                            int32_t *__restrict__ wid)
{
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        if (!(wxl[v] != 0ull && wxl[v] == wxg[v])) wid[v] = INT_MAX;
}

// new global suitors; which local proposers hold a local slot
__global__ void k_dist_update(int64_t nB, const unsigned long long *__restrict__ wxg, const int32_t *__restrict__ wid,
                              unsigned long long *__restrict__ gx, int32_t *__restrict__ gi,
                              const unsigned long long *__restrict__ sT, const int32_t *__restrict__ La, int32_t e0,
                              int32_t e1, int32_t p0, int32_t nPl, int32_t *__restrict__ hold)
{
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < 2 * nB; v += (int64_t)gridDim.x * blockDim.x) {
        gx[v] = wxg[v];
        gi[v] = wid[v] == INT_MAX ? -1 : wid[v];
        const unsigned long long s = sT[v];
        if (s) {
            const int e = (int)(uint32_t)s;
            if (e >= e0 && e < e1) hold[(v < nB ? 0 : nPl) + (La[e] - p0)] = e;
        }
    }
}

// a local proposer is active next round iff it holds a slot locally that is
// not the global suitor (displaced by another shard); count the active ones
__global__ void k_dist_active(int32_t nPl, int64_t nB, const int32_t *__restrict__ hold,
                              const int32_t *__restrict__ gi, const int32_t *__restrict__ Lb,
                              int32_t *__restrict__ act, unsigned long long *__restrict__ cnt)
{
    unsigned long long c = 0;
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < 2 * (int64_t)nPl;
         j += (int64_t)gridDim.x * blockDim.x) {
        const int e = hold[j];
        const int k = j < nPl ? 0 : 1;
        const int a = (e >= 0 && gi[k * nB + Lb[e]] != e) ? 1 : 0;
        act[j] = a;
        c += a;
    }
    for (int off = 16; off >= 1; off >>= 1) c += __shfl_down_sync(0xffffffffu, c, off);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(cnt, c);
}

__global__ void k_dist_mates(int64_t nB, int64_t nA, const int32_t *__restrict__ gi, const int32_t *__restrict__ La,
                             MatchParams P, int32_t *__restrict__ mateB)
{
    int32_t *mateA = slot_mates(P);
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < 2 * nB; v += (int64_t)gridDim.x * blockDim.x) {
        const int e = gi[v];
        mateB[v] = e;
        if (e >= 0) mateA[(v < nB ? 0 : nA) + La[e]] = e;
    }
}

__global__ void k_fill_i32(int64_t n, int32_t *__restrict__ x, int32_t v)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) x[i] = v;
}

// The final suitor of each target is its mate: mates of both sides and the
// B vertex of each matched A vertex (evaluate's input) from the target slots;
// proposers left unmatched were written by k_suitor.  Every slot is reset to
// empty for the next rounding (no separate reset pass), and the round's
// overlap / cardinality accumulators are zeroed (k_eval follows).
__device__ __forceinline__ void collect_body(const MatchParams &P, int64_t nT, int64_t nP, int fromB)
{
    if (blockIdx.x == 0 && threadIdx.x < 4) (&P.rd->overlap[0])[threadIdx.x] = 0ull; // overlap[2], card[2]
    if (P.qcnt && blockIdx.x == 0 && threadIdx.x < QBUF * NQ) P.qcnt[threadIdx.x * QSTRIDE] = 0; // next rounding
    int32_t *mateA = slot_mates(P);
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < P.ninst * nT;
         v += (int64_t)gridDim.x * blockDim.x) {
        const int k = (int)(v / nT);
        const int64_t t = v - k * nT;
        const unsigned long long s = P.suit[v];
        if (s) P.suit[v] = 0ull;
        const int e = s ? (int)(uint32_t)s : -1;
        if (!fromB) {             // targets are B vertices
            P.mateB[v] = e;
            if (e >= 0) {
                const int a = __ldg(P.La + e);
                mateA[k * nP + a] = e;
                set_mv(P.mvA, a, k, (int)t);
            }
        } else {                  // targets are A vertices
            mateA[v] = e;
            set_mv(P.mvA, t, k, e >= 0 ? __ldg(P.Lb + e) : -1);
            if (e >= 0) P.mateB[k * nP + __ldg(P.Lb + e)] = e;
        }
    }
}

// deferred evaluate: this round's mate slot (both instances) and mvA to -1
// (the collect pass then writes the matched entries)
__global__ void k_defer_fill(MatchParams P)
{
    pdl_wait();
    int32_t *mateA = slot_mates(P);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < P.nA; i += (int64_t)gridDim.x * blockDim.x) {
        mateA[i] = -1;
        mateA[P.nA + i] = -1;
        P.mvA[i] = make_int2(-1, -1);
    }
}

__global__ void k_collect(MatchParams P, int64_t nT, int64_t nP, int fromB)
{
    pdl_wait();
    collect_body(P, nT, nP, fromB);
}

__global__ void k_fill_slot(MatchParams P, int64_t n)
{
    int32_t *mateA = slot_mates(P);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        mateA[i] = -1;
}

// ---------------------------------------------------------- pointer rounds
__device__ int cand_A(const MatchParams &P, int k, int a)
{
    const double *x = xk(P, k);
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
    const double *x = xk(P, k);
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

__global__ void __launch_bounds__(256) k_pointer_rounds(MatchParams P)
{
    P.mateA = slot_mates(P);
    cg::grid_group grid = cg::this_grid();
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    const int64_t nA = P.nA, nB = P.nB;
    const int64_t NV = nA + nB;
    RoundDev *rd = P.rd;
    if (tid == 0) {
        for (int k = 0; k < 2; k++) rd->flag[0][k] = rd->flag[1][k] = 0;
    }
    for (int64_t v = tid; v < P.ninst * NV; v += nthr) {
        const int k = (int)(v / NV);
        const int64_t r = v - k * NV;
        if (r < nA) P.mateA[k * nA + r] = -1;
        else P.mateB[k * nB + (r - nA)] = -1;
    }
    grid.sync();
    for (int64_t v = tid; v < P.ninst * NV; v += nthr) {
        const int k = (int)(v / NV);
        const int64_t r = v - k * NV;
        if (r < nA) P.candA[k * nA + r] = cand_A(P, k, (int)r);
        else P.candB[k * nB + (r - nA)] = cand_B(P, k, (int)(r - nA));
    }
    grid.sync();
    for (int round = 0; round < P.max_rounds; round++) {
        const int par = round & 1;
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
            P.work[0] += f0;
            P.work[1] += f1;
        }
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
}

// ---------------------------------------------------------------- evaluate
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

struct EvalParams {
    int64_t nA;
    const int32_t *Lb;
    const double *w;
    const int32_t *mates; // [2 slots][2 instances][nA]; this round's slot is *wslot
    const int *wslot;
    const int2 *mvA;      // (M_y(i), M_z(i)) as B vertices (-1: unmatched)
    const unsigned long long *Bhash; // E_B membership set
    int Bhash_log;
    const int2 *pairs;    // undirected A edges (i < j)
    int64_t npairs;
    double *partial_w;    // [2][gridDim]
    RoundDev *rd;
};

// One block (the last one of k_eval to finish): finish the sums, score, select,
// best (Alg. 2 l.21-24).
__device__ void round_final_block(const EvalParams &P, const int32_t *mateA, int nblocks, int exact, double alpha,
                                  double beta, const int *p_dev, unsigned long long *work, double *sd)
{
    double wk[2] = {0.0, 0.0};
    for (int k = 0; k < 2; k++) {
        if (exact) {
            // oracle order: ascending edge id == ascending A vertex
            if (threadIdx.x == 0) {
                double s = 0.0;
                const int32_t *mA = mateA + (int64_t)k * P.nA;
                for (int64_t a = 0; a < P.nA; a++)
                    if (mA[a] >= 0) s = s + P.w[mA[a]];
                wk[k] = s;
            }
        } else {
            double s = 0.0;
            for (int i = threadIdx.x; i < nblocks; i += blockDim.x) s += __ldcg(P.partial_w + k * nblocks + i);
            s = block_sum<double>(s, sd);
            if (threadIdx.x == 0) wk[k] = s;
        }
    }
    if (threadIdx.x != 0) return;
    RoundDev *rd = P.rd;
    cualign_round_info &I = rd->info;
    const long long ov0 = (long long)*(volatile unsigned long long *)&rd->overlap[0];
    const long long ov1 = (long long)*(volatile unsigned long long *)&rd->overlap[1];
    const int32_t p = *p_dev;
    I.iter = p;
    I.weight_y = wk[0];
    I.weight_z = wk[1];
    I.overlap_y = ov0;
    I.overlap_z = ov1;
    I.card_y = (int32_t)*(volatile unsigned long long *)&rd->card[0];
    I.card_z = (int32_t)*(volatile unsigned long long *)&rd->card[1];
    I.score_y = alpha * wk[0] + beta * (double)ov0;
    I.score_z = alpha * wk[1] + beta * (double)ov1;
    unsigned long long w0 = 0, w1 = 0;
    for (int i = 0; i < WORK_SPREAD; i++) {
        w0 += work[i * WORK_STRIDE];
        w1 += work[i * WORK_STRIDE + 1];
        work[i * WORK_STRIDE] = 0ull; // ready for the next rounding
        work[i * WORK_STRIDE + 1] = 0ull;
    }
    I.rounds_y = (int32_t)w0;
    I.rounds_z = (int32_t)w1;
    const int src = (I.score_y >= I.score_z) ? 0 : 1;
    I.source = src;
    I.score = src ? I.score_z : I.score_y;
    I.improved = 0;
    const int ws = rd->wslot;
    if (I.score > rd->best_score) {
        rd->best_score = I.score;
        rd->best_iter = p;
        rd->best_slot = ws; // bestM = this round's M_src, kept in place
        rd->best_source = src;
        I.improved = 1;
    }
    I.best_score = rd->best_score;
    I.best_iter = rd->best_iter;
    rd->improved = I.improved;
    rd->source = src;
    rd->last_slot = ws;
    rd->wslot = 1 - rd->best_slot;
}

// Evaluate M_y and M_z.  weight: partial sums per block over a fixed
// partition of the A vertices (deterministic); cardinality and overlap:
// integer atomics (exact).  Overlap by PAPER.md:60: one thread per undirected
// A edge {i, j}; it counts when both ends are matched and (M(i), M(j)) is an
// edge of B (one probe of the E_B membership set, ~1 dependent load instead of
// a ~5-load binary search in B's row of M(i)) -- balanced whatever the degree
// of i.  The last block to finish runs the final reduction.
//
// COLLECT: the Suitor's collect pass (k_collect) runs first inside this kernel
// -- the grid is one wave (every block resident), so a grid-wide barrier
// (arrival counter in RoundDev, reset by the final block after every block
// has left it) separates the two instead of a kernel boundary.
template <bool COLLECT>
__global__ void __launch_bounds__(EVAL_BS)
k_eval(EvalParams P, int exact, double alpha, double beta, const int *p_dev, unsigned long long *work,
       MatchParams M, int64_t nT, int64_t nP, int fromB)
{
    pdl_wait();
    __shared__ double sd[32];
    __shared__ unsigned long long su[32];
    __shared__ bool last;
    if (COLLECT) {
        collect_body(M, nT, nP, fromB);
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            atomicAdd(&P.rd->gbar, 1u);
            while (*(volatile unsigned int *)&P.rd->gbar < gridDim.x) __nanosleep(64);
            __threadfence();
        }
        __syncthreads();
    }
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    const int32_t *mateA = P.mates + (int64_t)(*(volatile const int *)P.wslot) * 2 * P.nA;
    double wsum[2] = {0.0, 0.0};
    unsigned long long ov[2] = {0, 0}, card[2] = {0, 0};
    for (int64_t i = tid; i < P.nA; i += nthr) {
        const int e0 = mateA[i], e1 = mateA[P.nA + i];
        if (e0 >= 0) {
            wsum[0] += P.w[e0];
            card[0]++;
        }
        if (e1 >= 0) {
            wsum[1] += P.w[e1];
            card[1]++;
        }
    }
    // EVAL_U pairs per thread and pass, each level of the dependent chain
    // (pair -> mates -> M(i), M(j) -> probe) issued for all of them together
    constexpr int EVAL_U = 4;
    for (int64_t base = tid; base < P.npairs; base += nthr * EVAL_U) {
        int2 ij[EVAL_U];
        int2 mi[EVAL_U], mj[EVAL_U]; // (M_y, M_z) of i and of j as B vertices
#pragma unroll
        for (int u = 0; u < EVAL_U; u++) {
            const int64_t q = base + u * nthr;
            ij[u] = q < P.npairs ? __ldg(P.pairs + q) : make_int2(-1, -1);
        }
        // both instances' images of i and j: one 8-byte gather each (pairs
        // are sorted by i, so the i gathers mostly hit the same line; j is
        // gathered only when i is matched in some instance)
#pragma unroll
        for (int u = 0; u < EVAL_U; u++) mi[u] = ij[u].x >= 0 ? P.mvA[ij[u].x] : make_int2(-1, -1);
#pragma unroll
        for (int u = 0; u < EVAL_U; u++)
            mj[u] = (mi[u].x >= 0 || mi[u].y >= 0) ? P.mvA[ij[u].y] : make_int2(-1, -1);
#pragma unroll
        for (int u = 0; u < EVAL_U; u++) {
            // M_y and M_z agree on most vertices (94 % on O): when both
            // instances ask the same question, probe once
            const bool hy = mi[u].x >= 0 && mj[u].x >= 0 &&
                            bhash_has(P.Bhash, P.Bhash_log, bhash_key(mi[u].x, mj[u].x));
            const bool same = mi[u].x == mi[u].y && mj[u].x == mj[u].y;
            const bool hz = same ? hy
                                 : (mi[u].y >= 0 && mj[u].y >= 0 &&
                                    bhash_has(P.Bhash, P.Bhash_log, bhash_key(mi[u].y, mj[u].y)));
            ov[0] += hy;
            ov[1] += hz;
        }
    }
    for (int k = 0; k < 2; k++) {
        const double bw = block_sum<double>(wsum[k], sd);
        if (threadIdx.x == 0) P.partial_w[k * gridDim.x + blockIdx.x] = bw;
        const unsigned long long bo = block_sum<unsigned long long>(ov[k], su);
        if (threadIdx.x == 0 && bo) atomicAdd(&P.rd->overlap[k], bo);
        const unsigned long long bc = block_sum<unsigned long long>(card[k], su);
        if (threadIdx.x == 0 && bc) atomicAdd(&P.rd->card[k], bc);
    }
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(&P.rd->done, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    round_final_block(P, mateA, gridDim.x, exact, alpha, beta, p_dev, work, sd);
    if (threadIdx.x == 0) {
        P.rd->done = 0u;
        if (COLLECT) P.rd->gbar = 0u; // every block is past the barrier (it counted in `done`)
    }
}

// Schedules whose kernels leave complete mate arrays (pointer rounds, the
// sharded merge): (M_y(i), M_z(i)) as B vertices from this round's slot, and
// the round's overlap / cardinality accumulators zeroed (k_eval follows).
__global__ void k_mate_vertex(int64_t nA, const int32_t *__restrict__ mates, const int *__restrict__ wslot,
                              const int32_t *__restrict__ Lb, int2 *__restrict__ mvA, RoundDev *rd)
{
    pdl_wait();
    if (blockIdx.x == 0 && threadIdx.x < 4) (&rd->overlap[0])[threadIdx.x] = 0ull; // overlap[2], card[2]
    const int32_t *mA = mates + (int64_t)(*(volatile const int *)wslot) * 2 * nA;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nA; i += (int64_t)gridDim.x * blockDim.x) {
        const int e0 = mA[i], e1 = mA[nA + i];
        mvA[i] = make_int2(e0 >= 0 ? __ldg(Lb + e0) : -1, e1 >= 0 ? __ldg(Lb + e1) : -1);
    }
}

__global__ void k_maxdeg(int64_t nA, const int64_t *__restrict__ Arow, int64_t nB,
                         const int64_t *__restrict__ Bptr, unsigned long long *out)
{
    unsigned long long ma = 0, mb = 0;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < nA + nB;
         v += (int64_t)gridDim.x * blockDim.x) {
        if (v < nA) {
            const unsigned long long d = (unsigned long long)(Arow[v + 1] - Arow[v]);
            ma = d > ma ? d : ma;
        } else {
            const unsigned long long d = (unsigned long long)(Bptr[v - nA + 1] - Bptr[v - nA]);
            mb = d > mb ? d : mb;
        }
    }
    // warp max first: one atomic per warp
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
        const unsigned long long oa = __shfl_xor_sync(0xffffffffu, ma, off);
        const unsigned long long ob = __shfl_xor_sync(0xffffffffu, mb, off);
        ma = oa > ma ? oa : ma;
        mb = ob > mb ? ob : mb;
    }
    if ((threadIdx.x & 31) == 0) {
        if (ma) atomicMax(out, ma);
        if (mb) atomicMax(out + 1, mb);
    }
}

MatchParams base_params(cualign_bp *h)
{
    MatchParams P{};
    P.nA = h->L.nA;
    P.nB = h->L.nB;
    const int64_t mr = (int64_t)h->L.nA + h->L.nB + 4;
    P.max_rounds = (int)(mr > (1 << 30) ? (1 << 30) : mr);
    P.La = h->L.La;
    P.Lb = h->L.Lb;
    P.Arow = h->L.Arow;
    P.Bptr = h->L.Bptr;
    P.Bedge = h->L.Bedge;
    P.candA = h->candA;
    P.candB = h->candB;
    P.suit = h->suit;
    P.mates = h->mates;
    P.wslot = &h->rd->wslot;
    P.mateB = h->mateB;
    P.mvA = h->mvA;
    P.rd = h->rd;
    P.work = h->match_work;
    return P;
}

// Run the matching of P.ninst instances into this round's mate slot.
// Suitor: k_suitor (exhausted proposers) + k_collect (everything held in a
// target slot; resets the slots) leave the mates of both sides, mvA and zeroed
// round accumulators -- ready for k_eval.  Pointer rounds leave complete mate
// arrays (k_mate_vertex prepares evaluate).
cualign_status run_matching(cualign_bp *h, MatchParams &P, bool collect_in_eval = false)
{
    const int64_t nA = h->L.nA, nB = h->L.nB;
    if (h->flags & CUALIGN_FLAG_MATCH_ROUNDS) {
        KScope ks(h, CUALIGN_K_MATCH);
        // cooperative launch through cudaLaunchKernelEx: capturable into a graph
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(h->match_grid);
        cfg.blockDim = dim3(256);
        cfg.stream = h->stream;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeCooperative;
        attr[0].val.cooperative = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        CA_CUDA(cudaLaunchKernelEx(&cfg, k_pointer_rounds, P));
        return CUALIGN_OK;
    }
    const bool fromB = h->propose_from_b;
    P.propose_from_b = fromB ? 1 : 0;
    const int64_t nP = fromB ? nB : nA, nT = fromB ? nA : nB;
    const int64_t slots = P.ninst * nP;
    static const bool dbg_env = probe_knob("CUALIGN_MATCH_DEBUG", 0) != 0;
    const bool dbg = dbg_env && !h->capturing;
    unsigned long long *dbuf = nullptr;
    if (dbg) {
        CA_CUDA(cudaMalloc(&dbuf, 8 * sizeof(unsigned long long)));
        CA_CUDA(cudaMemsetAsync(dbuf, 0, 8 * sizeof(unsigned long long), h->stream));
        P.dbg = dbuf;
    }
    static const int two_env = probe_knob("CUALIGN_SUITOR_QROUNDS", 1);
    const bool two = two_env && !fromB && h->max_deg_a <= SUITOR_ROUNDS_MAXDEG && h->squeue && !dbg;
    static const int chain_mode = probe_knob("CUALIGN_SUITOR_CHAIN", 0);
    if (two && slots > 0 && chain_mode) {
        P.qcnt = h->qcnt;
        KScope ks(h, CUALIGN_K_MATCH);
        CA_CUDA(launch_pdl(k_propose_chain<6>, dim3(grid_for(slots, 256, 1 << 30)), dim3(256), 0, h->stream, P));
        CA_CUDA(cudaGetLastError());
    } else if (two && slots > 0) {
        // proposal rounds (see k_propose_round), then the chain form for
        // whatever is still queued
        P.qcnt = h->qcnt;
        KScope ks(h, CUALIGN_K_MATCH);
        const int64_t qc = h->qcap, cs = (int64_t)NQ * QSTRIDE;
        // 3 rounds, measured in the bench's window (p = 6-25 on O): matching
        // 0.206 / 0.165 / 0.148 / 0.158 / 0.176 ms with 1 / 2 / 3 / 4 / 6
        // rounds (at p = 80 alone 2 rounds were best: 0.112 vs 0.121 ms; early
        // BP iterations displace far more proposers).  Each round costs ~9
        // dependent memory round trips even nearly empty; the chain form takes
        // the rest.  Rejected: a persistent kernel looping over rounds with
        // grid barriers until the queue is short (0.162 / 0.143 ms), rounds
        // that skip once the queue is short (0.158 / 0.126 ms).
        static const int nrounds = probe_knob("CUALIGN_SUITOR_ROUNDS", 3);
        static const int first_u = probe_knob("CUALIGN_SUITOR_FIRST_U", 6);
        if (first_u == 9)
            CA_CUDA(launch_pdl(k_propose_first<9>, dim3(grid_for(slots, 256, 1 << 30)), dim3(256), 0, h->stream, P,
                               h->squeue + 1 * NQ * qc, h->qcnt + 1 * cs, qc));
        else if (first_u == 18)
            CA_CUDA(launch_pdl(k_propose_first<18>, dim3(grid_for(slots, 256, 1 << 30)), dim3(256), 0, h->stream, P,
                               h->squeue + 1 * NQ * qc, h->qcnt + 1 * cs, qc));
        else
            CA_CUDA(launch_pdl(k_propose_first<6>, dim3(grid_for(slots, 256, 1 << 30)), dim3(256), 0, h->stream, P,
                               h->squeue + 1 * NQ * qc, h->qcnt + 1 * cs, qc));
        for (int r = 1; r <= nrounds; r++) {
            const int bi = r % QBUF, bo = (r + 1) % QBUF, bc = (r + 2) % QBUF;
            CA_CUDA(launch_pdl(k_propose_round<6>, dim3(h->qr_grid), dim3(256), 0, h->stream, P,
                               (const int32_t *)(h->squeue + bi * NQ * qc), (const int *)(h->qcnt + bi * cs),
                               h->squeue + bo * NQ * qc, h->qcnt + bo * cs, h->qcnt + bc * cs, qc));
        }
        const int bl = (nrounds + 1) % QBUF;
        CA_CUDA(launch_pdl(k_suitor_q<4, 5, 8>, dim3(h->q2_grid), dim3(128), 0, h->stream, P,
                           (const int32_t *)(h->squeue + bl * NQ * qc), (const int *)(h->qcnt + bl * cs), qc));
        CA_CUDA(cudaGetLastError());
    } else if (slots > 0) {
        KScope ks(h, CUALIGN_K_MATCH);
        const int64_t dmax = fromB ? h->max_deg_b : h->max_deg_a;
        static const int genv = probe_knob("CUALIGN_SUITOR_G", 0);
        // tile width: G lanes x U edges cover a typical proposer list in one pass
        const int G = genv ? genv : (dmax > 64 ? 32 : (dmax > 24 ? 16 : (dmax > 20 ? 8 : 4)));
        if (G == 32) CA_CUDA(launch_pdl(k_suitor<32, 2>, dim3(grid_for(slots * 32, 128, 1 << 30)), dim3(128), 0, h->stream, P));
        else if (G == 16) CA_CUDA(launch_pdl(k_suitor<16, 2>, dim3(grid_for(slots * 16, 128, 1 << 30)), dim3(128), 0, h->stream, P));
        else if (G == 8) CA_CUDA(launch_pdl(k_suitor<8, 3>, dim3(grid_for(slots * 8, 128, 1 << 30)), dim3(128), 0, h->stream, P));
        else if (G == 2) CA_CUDA(launch_pdl(k_suitor<2, 9>, dim3(grid_for(slots * 2, 128, 1 << 30)), dim3(128), 0, h->stream, P));
        else if (G == 1) CA_CUDA(launch_pdl(k_suitor<1, 8>, dim3(grid_for(slots, 128, 1 << 30)), dim3(128), 0, h->stream, P));
        else {
            // resident blocks per SM (register cap), probe build knob:
            // default 12 blocks of 128 (40 registers): 0.142 ms vs 0.175 ms
            // uncapped (66 registers, 8 blocks) on O -- latency-bound, more
            // resident proposer tiles win over a few spilled registers
            static const int minb = probe_knob("CUALIGN_SUITOR_MINB", 12);
            const int grid = grid_for(slots * 4, 128, 1 << 30);
            static const int pers = probe_knob("CUALIGN_SUITOR_PERSIST", 0);
            if (pers) {
                int occ = 0;
                if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_suitor_persistent<4, 5, 12>, 128, 0) !=
                        cudaSuccess || occ < 1)
                    occ = 1;
                (void)cudaGetLastError();
                k_suitor_persistent<4, 5, 12><<<grid_for(slots * 4, 128, (int64_t)occ * h->num_sms), 128, 0,
                                                h->stream>>>(P);
            } else if (minb >= 16) CA_CUDA(launch_pdl(k_suitor<4, 5, false, 16>, dim3(grid), dim3(128), 0, h->stream, P));
            else if (minb >= 12) CA_CUDA(launch_pdl(k_suitor<4, 5, false, 12>, dim3(grid), dim3(128), 0, h->stream, P));
            else if (minb >= 10) CA_CUDA(launch_pdl(k_suitor<4, 5, false, 10>, dim3(grid), dim3(128), 0, h->stream, P));
            else CA_CUDA(launch_pdl(k_suitor<4, 5>, dim3(grid), dim3(128), 0, h->stream, P));
        }
        CA_CUDA(cudaGetLastError());
    }
    if (dbg) {
        unsigned long long d[8];
        CA_CUDA(cudaMemcpyAsync(d, dbuf, sizeof(d), cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream));
        fprintf(stderr, "[suitor] tiles=%lld max_scans=%llu total_scans=%llu tiles>8=%llu tiles>64=%llu max_props=%llu\n",
                (long long)slots, d[0], d[1], d[2], d[3], d[4]);
        cudaFree(dbuf);
    }
    if (!collect_in_eval) { // else the collect pass opens k_eval<true> (match_evaluate)
        KScope ks(h, CUALIGN_K_MATCHAUX);
        CA_CUDA(launch_pdl(k_collect, dim3(grid_for(P.ninst * nT > 0 ? P.ninst * nT : 1, 256, h->num_sms * 8)),
                           dim3(256), 0, h->stream, P, nT, nP, fromB ? 1 : 0));
        CA_CUDA(cudaGetLastError());
    }
    return CUALIGN_OK;
}

// (M_y(i), M_z(i)) for evaluate from complete mate arrays (pointer rounds,
// sharded merge)
cualign_status prep_eval_from_mates(cualign_bp *h)
{
    KScope ks(h, CUALIGN_K_MATCHAUX);
    const int64_t nA = h->L.nA;
    CA_CUDA(launch_pdl(k_mate_vertex, dim3(grid_for(nA > 0 ? nA : 1, 256, h->num_sms * 4)), dim3(256), 0, h->stream,
                       nA, (const int32_t *)h->mates, (const int *)&h->rd->wslot, (const int32_t *)h->L.Lb, h->mvA,
                       h->rd));
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

} // namespace

cualign_status match_setup(cualign_bp *h)
{
    const size_t nA = (size_t)h->L.nA, nB = (size_t)h->L.nB;
    const size_t nmax = nA > nB ? nA : nB;
    CA_TRY(dalloc(h, &h->candA, 2 * nA + 1));
    CA_TRY(dalloc(h, &h->candB, 2 * nB + 1));
    CA_TRY(dalloc(h, &h->suit, 2 * nmax + 1));
    CA_TRY(dalloc(h, &h->mates, 4 * nA + 1));
    CA_TRY(dalloc(h, &h->mvA, nA + 1));
    CA_TRY(dalloc(h, &h->mateB, 2 * nB + 1));
    CA_TRY(dalloc(h, &h->rd, 1));
    CA_TRY(dalloc(h, &h->match_work, 2 * WORK_SPREAD * WORK_STRIDE)); // 2 sets: deferred evaluate
    {
        RoundDev r0;
        memset(&r0, 0, sizeof(r0));
        r0.wslot = 1; // slot 0 "holds" the empty bestM (best_iter = 0)
        CA_CUDA(cudaMemcpyAsync(h->rd, &r0, sizeof(RoundDev), cudaMemcpyHostToDevice, h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream)); // r0 is a stack object
    }
    CA_CUDA(cudaMemsetAsync(h->suit, 0, sizeof(unsigned long long) * (2 * nmax + 1), h->stream));
    CA_CUDA(cudaMemsetAsync(h->mates, 0xff, sizeof(int32_t) * (4 * nA + 1), h->stream));
    CA_CUDA(cudaMemsetAsync(h->mateB, 0xff, sizeof(int32_t) * (2 * nB + 1), h->stream));
    CA_CUDA(cudaMemsetAsync(h->match_work, 0, sizeof(unsigned long long) * 2 * WORK_SPREAD * WORK_STRIDE, h->stream));
    {
        KScope ks(h, CUALIGN_K_INIT);
        unsigned long long md[2] = {0, 0};
        k_maxdeg<<<grid_for((int64_t)(nA + nB), 256, h->num_sms * 8), 256, 0, h->stream>>>(
            (int64_t)nA, h->L.Arow, (int64_t)nB, h->L.Bptr, h->match_work);
        CA_CUDA(cudaGetLastError());
        CA_CUDA(cudaMemcpyAsync(md, h->match_work, sizeof(md), cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaMemsetAsync(h->match_work, 0, 2 * sizeof(unsigned long long), h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream));
        h->max_deg_a = (int64_t)md[0];
        h->max_deg_b = (int64_t)md[1];
        h->propose_from_b = h->max_deg_b < h->max_deg_a;
    }
    int occ = 0;
    CA_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pointer_rounds, 256, 0));
    if (occ < 1) occ = 1;
    int64_t want = ((int64_t)2 * (nA + nB) + 255) / 256;
    int64_t cap = (int64_t)occ * h->num_sms;
    h->match_grid = (int)(want < 1 ? 1 : (want > cap ? cap : want));
    {
        // one wave of k_eval (every block resident at once)
        int occ = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_eval<false>, EVAL_BS, 0) != cudaSuccess || occ < 1)
            occ = 1;
        (void)cudaGetLastError();
        h->eval_grid = grid_for(h->nApairs > (int64_t)nA ? h->nApairs : (int64_t)nA, EVAL_BS, h->num_sms * occ);
        // k_eval<true> holds a grid barrier: exactly one wave of its own occupancy
        int occc = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occc, k_eval<true>, EVAL_BS, 0) != cudaSuccess || occc < 1)
            occc = 1;
        (void)cudaGetLastError();
        h->evalc_grid = grid_for(std::max<int64_t>(std::max<int64_t>(h->nApairs, (int64_t)nA), 2 * (int64_t)nmax), EVAL_BS,
                                 h->num_sms * occc);
    }
    CA_TRY(dalloc(h, &h->partial_w, (size_t)2 * std::max(h->eval_grid, h->evalc_grid)));
    {
        // Suitor-round queues: sub-queue q collects the pushes of the
        // phase-1 warps w with w mod NQ = q, <= 32 per warp
        const int64_t nwarps = ((int64_t)2 * nA + 31) / 32;
        h->qcap = 32 * ((nwarps + NQ - 1) / NQ);
        CA_TRY(dalloc(h, &h->squeue, (size_t)(QBUF * NQ * h->qcap)));
        CA_TRY(dalloc(h, &h->qcnt, (size_t)QBUF * NQ * QSTRIDE));
        CA_CUDA(cudaMemsetAsync(h->qcnt, 0, sizeof(int) * QBUF * NQ * QSTRIDE, h->stream));
        int occr = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occr, k_propose_round<6>, 256, 0) != cudaSuccess ||
            occr < 1)
            occr = 1;
        (void)cudaGetLastError();
        h->qr_grid = occr * h->num_sms;
        int occ2 = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, k_suitor_q<4, 5, 8>, 128, 0) != cudaSuccess ||
            occ2 < 1)
            occ2 = 1;
        (void)cudaGetLastError();
        h->q2_grid = occ2 * h->num_sms;
    }
    return CUALIGN_OK;
}

static cualign_status evaluate_impl(cualign_bp *h, const MatchParams *Pc);

cualign_status match_evaluate(cualign_bp *h) { return evaluate_impl(h, nullptr); }

// Deferred-evaluate rounding (pipelined graphs, DESIGN.md "Step graph and
// schedule"): the matching of this round with proposal counters in `set`;
// the collect pass waits for `before_collect` (the previous round's
// evaluate, which picks this round's mate slot and reads mvA), presets the
// slot and mvA, then writes the matched entries and resets the target slots.
cualign_status match_round_deferred(cualign_bp *h, int set, cudaEvent_t before_collect)
{
    MatchParams P = base_params(h);
    P.ninst = 2;
    P.x0 = h->yc;
    P.x1 = h->zc;
    P.defer = 1;
    P.work = h->match_work + (int64_t)set * WORK_SPREAD * WORK_STRIDE;
    CA_TRY(run_matching(h, P, true)); // proposals only: the collect pass follows here
    if (before_collect) CA_CUDA(cudaStreamWaitEvent(h->stream, before_collect, 0));
    KScope ks(h, CUALIGN_K_MATCHAUX);
    const bool fromB = P.propose_from_b != 0;
    const int64_t nT = fromB ? h->L.nA : h->L.nB, nP = fromB ? h->L.nB : h->L.nA;
    k_defer_fill<<<grid_for(h->L.nA > 0 ? h->L.nA : 1, 256, h->num_sms * 8), 256, 0, h->stream>>>(P);
    CA_CUDA(cudaGetLastError());
    CA_CUDA(launch_pdl(k_collect, dim3(grid_for(P.ninst * nT > 0 ? P.ninst * nT : 1, 256, h->num_sms * 8)),
                       dim3(256), 0, h->stream, P, nT, nP, fromB ? 1 : 0));
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

// Its evaluate (one step later): k_eval without the collect pass, over the
// same block partition as k_eval<true> (evalc_grid), so the weights carry the
// same bits as in the other schedules; proposal counters of `set`.
cualign_status eval_round_deferred(cualign_bp *h, int set)
{
    EvalParams E{};
    E.nA = h->L.nA;
    E.Lb = h->L.Lb;
    E.w = h->L.w;
    E.mates = h->mates;
    E.wslot = &h->rd->wslot;
    E.mvA = h->mvA;
    E.Bhash = h->Bhash;
    E.Bhash_log = h->Bhash_log;
    E.pairs = h->Apairs;
    E.npairs = h->nApairs;
    E.partial_w = h->partial_w;
    E.rd = h->rd;
    KScope ks(h, CUALIGN_K_EVAL);
    const int exact = (h->flags & CUALIGN_FLAG_EXACT) ? 1 : 0;
    const int *pd = (const int *)(h->round_p ? h->round_p : h->p_dev);
    CA_CUDA(launch_pdl(k_eval<false>, dim3(h->evalc_grid), dim3(EVAL_BS), 0, h->stream, E, exact, h->alpha, h->beta, pd,
                       h->match_work + (int64_t)set * WORK_SPREAD * WORK_STRIDE, MatchParams{}, (int64_t)0,
                       (int64_t)0, 0));
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

// whether this handle's rounding can run deferred (Suitor proposal rounds)
bool can_defer_eval(const cualign_bp *h)
{
    return !h->propose_from_b && h->max_deg_a <= SUITOR_ROUNDS_MAXDEG && h->squeue &&
           !(h->flags & (CUALIGN_FLAG_ROUND_DAMPED | CUALIGN_FLAG_MATCH_ROUNDS)) && h->world == 1;
}

cualign_status match_round(cualign_bp *h)
{
    MatchParams P = base_params(h);
    const bool damped = (h->flags & CUALIGN_FLAG_ROUND_DAMPED) != 0;
    P.ninst = 2;
    P.x0 = damped ? h->yp : h->yc;
    P.x1 = damped ? h->zp : h->zc;
    if (h->flags & CUALIGN_FLAG_MATCH_ROUNDS) {
        CA_TRY(run_matching(h, P));
        CA_TRY(prep_eval_from_mates(h));
        return match_evaluate(h);
    }
    if (h->probe_no_eval) { // timing probe (probe build): collect only, no evaluate (wrong round info)
        CA_TRY(run_matching(h, P, false));
        return CUALIGN_OK;
    }
    CA_TRY(run_matching(h, P, true));
    return evaluate_impl(h, &P);
}

// ------------------------------------------------ sharded rounding (NEXT-1)
// Deferred acceptance in rounds across shards.  Every
// shard proposes only from its own A rows (so it needs y^c, z^c only on its
// own edges -- no all-gather of the messages); the targets' suitors are kept
// replicated as (weight bits, edge id) per B vertex.  A round: each shard runs
// the Suitor kernel for its active proposers against slots initialised with
// the global suitors (local displacement chains resolve inside the round),
// then the local winners are merged: all-reduce MAX of the weight bits, then
// all-reduce MIN of the edge id among the shards holding that weight (lowest
// index wins, Z7).  A proposer whose slot went to another shard is active in
// the next round; rounds end when no shard has an active proposer.  The
// stable matching under one strict edge order is unique, so the result is the
// single-GPU (greedy) matching bit for bit; evaluation is then replicated.
static MatchParams dist_params(cualign_bp *h)
{
    MatchParams P = base_params(h);
    const bool damped = (h->flags & CUALIGN_FLAG_ROUND_DAMPED) != 0;
    P.ninst = 2;
    P.x0 = damped ? h->yp : h->yc;
    P.x1 = damped ? h->zp : h->zc;
    P.propose_from_b = 0;
    P.p0 = h->a0;
    P.nPl = h->a1 - h->a0;
    P.e0 = (int32_t)h->e0;
    P.e1 = (int32_t)h->e1;
    P.gx = h->dist_gx;
    P.gi = h->dist_gi;
    P.act = h->dist_act;
    return P;
}

cualign_status dist_match_begin(cualign_bp *h)
{
    const size_t nB = (size_t)h->L.nB, nPl = (size_t)(h->a1 - h->a0);
    if (!h->dist_gx) {
        CA_TRY(dalloc(h, &h->dist_gx, 2 * nB + 1));
        CA_TRY(dalloc(h, &h->dist_wxl, 2 * nB + 1));
        CA_TRY(dalloc(h, &h->dist_wxg, 2 * nB + 1));
        CA_TRY(dalloc(h, &h->dist_gi, 2 * nB + 1));
        CA_TRY(dalloc(h, &h->dist_wid, 2 * nB + 1));
        CA_TRY(dalloc(h, &h->dist_hold, 2 * nPl + 1));
        CA_TRY(dalloc(h, &h->dist_act, 2 * nPl + 1));
        CA_TRY(dalloc(h, &h->dist_cnt, 1));
        CA_CUDA(cudaHostAlloc((void **)&h->dist_cnt_host, sizeof(unsigned long long) * 16, cudaHostAllocDefault));
    }
    const int G = h->num_sms * 8;
    CA_CUDA(cudaMemsetAsync(h->match_work, 0, WORK_SPREAD * WORK_STRIDE * sizeof(unsigned long long), h->stream));
    CA_CUDA(cudaMemsetAsync(h->dist_gx, 0, sizeof(unsigned long long) * (2 * nB + 1), h->stream));
    k_fill_i32<<<grid_for((int64_t)(2 * nB + 1), 256, G), 256, 0, h->stream>>>((int64_t)(2 * nB + 1), h->dist_gi, -1);
    k_fill_i32<<<grid_for((int64_t)(2 * nPl + 1), 256, G), 256, 0, h->stream>>>((int64_t)(2 * nPl + 1), h->dist_act, 1);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status dist_match_local(cualign_bp *h)
{
    MatchParams P = dist_params(h);
    const int64_t nB = h->L.nB, slots = 2 * (int64_t)P.nPl;
    const int G = h->num_sms * 8;
    KScope ks(h, CUALIGN_K_MATCH);
    k_dist_init_slots<<<grid_for(2 * nB, 256, G), 256, 0, h->stream>>>(2 * nB, h->dist_gx, h->dist_gi, h->suit);
    if (slots > 0) {
        const int64_t dmax = h->max_deg_a;
        if (dmax > 64) k_suitor<32, 2, true><<<grid_for(slots * 32, 128, 1 << 30), 128, 0, h->stream>>>(P);
        else if (dmax > 24) k_suitor<16, 2, true><<<grid_for(slots * 16, 128, 1 << 30), 128, 0, h->stream>>>(P);
        else if (dmax > 20) k_suitor<8, 3, true><<<grid_for(slots * 8, 128, 1 << 30), 128, 0, h->stream>>>(P);
        else k_suitor<4, 5, true, 12><<<grid_for(slots * 4, 128, 1 << 30), 128, 0, h->stream>>>(P);
    }
    k_dist_pack<<<grid_for(2 * nB, 256, G), 256, 0, h->stream>>>(nB, h->suit, h->dist_gx, h->dist_gi, P.x0, P.x1,
                                                                 h->dist_wxl, h->dist_wxg, h->dist_wid);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status dist_match_cand(cualign_bp *h)
{
    const int64_t n = 2 * (int64_t)h->L.nB;
    k_dist_cand<<<grid_for(n, 256, h->num_sms * 8), 256, 0, h->stream>>>(n, h->dist_wxl, h->dist_wxg, h->dist_wid);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status dist_match_update(cualign_bp *h)
{
    const int64_t nB = h->L.nB;
    const int32_t nPl = h->a1 - h->a0;
    const int G = h->num_sms * 8;
    k_fill_i32<<<grid_for(2 * (int64_t)nPl + 1, 256, G), 256, 0, h->stream>>>(2 * (int64_t)nPl + 1, h->dist_hold, -1);
    k_dist_update<<<grid_for(2 * nB, 256, G), 256, 0, h->stream>>>(nB, h->dist_wxg, h->dist_wid, h->dist_gx,
                                                                   h->dist_gi, h->suit, h->L.La, (int32_t)h->e0,
                                                                   (int32_t)h->e1, h->a0, nPl, h->dist_hold);
    CA_CUDA(cudaMemsetAsync(h->dist_cnt, 0, sizeof(unsigned long long), h->stream));
    if (nPl > 0)
        k_dist_active<<<grid_for(2 * (int64_t)nPl, 256, G), 256, 0, h->stream>>>(nPl, nB, h->dist_hold, h->dist_gi,
                                                                                 h->L.Lb, h->dist_act, h->dist_cnt);
    CA_CUDA(cudaGetLastError());
    return CUALIGN_OK;
}

cualign_status dist_match_finish(cualign_bp *h)
{
    const int64_t nA = h->L.nA, nB = h->L.nB;
    {
        KScope ks(h, CUALIGN_K_MATCHAUX);
        MatchParams P = base_params(h);
        k_fill_slot<<<grid_for(2 * nA + 1, 256, h->num_sms * 8), 256, 0, h->stream>>>(P, 2 * nA);
        if (nB)
            k_dist_mates<<<grid_for(2 * nB, 256, h->num_sms * 8), 256, 0, h->stream>>>(nB, nA, h->dist_gi, h->L.La,
                                                                                       P, h->mateB);
        CA_CUDA(cudaGetLastError());
    }
    CA_TRY(prep_eval_from_mates(h));
    return match_evaluate(h);
}

// a8 (evaluate + best) of this round's mates (slot rd->wslot) and mvA; the
// final block records bestM by slot (no copy).  Pc: the Suitor's collect
// pass runs at the start of the same kernel (k_eval<true>).
static cualign_status evaluate_impl(cualign_bp *h, const MatchParams *Pc)
{
    EvalParams E{};
    E.nA = h->L.nA;
    E.Lb = h->L.Lb;
    E.w = h->L.w;
    E.mates = h->mates;
    E.wslot = &h->rd->wslot;
    E.mvA = h->mvA;
    E.Bhash = h->Bhash;
    E.Bhash_log = h->Bhash_log;
    E.pairs = h->Apairs;
    E.npairs = h->nApairs;
    E.partial_w = h->partial_w;
    E.rd = h->rd;
    {
        KScope ks(h, CUALIGN_K_EVAL);
        const int exact = (h->flags & CUALIGN_FLAG_EXACT) ? 1 : 0;
        const int *pd = (const int *)(h->round_p ? h->round_p : h->p_dev);
        if (Pc) {
            const bool fromB = Pc->propose_from_b != 0;
            const int64_t nT = fromB ? h->L.nA : h->L.nB, nP = fromB ? h->L.nB : h->L.nA;
            CA_CUDA(launch_pdl(k_eval<true>, dim3(h->evalc_grid), dim3(EVAL_BS), 0, h->stream, E, exact, h->alpha,
                               h->beta, pd, h->match_work, *Pc, nT, nP, fromB ? 1 : 0));
        } else {
            CA_CUDA(launch_pdl(k_eval<false>, dim3(h->eval_grid), dim3(EVAL_BS), 0, h->stream, E, exact, h->alpha,
                               h->beta, pd, h->match_work, MatchParams{}, (int64_t)0, (int64_t)0, 0));
        }
        CA_CUDA(cudaGetLastError());
    }
    return CUALIGN_OK;
}

cualign_status match_standalone(cualign_bp *h, const double *x_dev, int32_t *rounds)
{
    MatchParams P = base_params(h);
    P.ninst = 1;
    P.x0 = x_dev;
    P.x1 = x_dev;
    CA_CUDA(cudaMemsetAsync(h->match_work, 0, WORK_SPREAD * WORK_STRIDE * sizeof(unsigned long long), h->stream));
    CA_TRY(run_matching(h, P));
    if (rounds) {
        std::vector<unsigned long long> w(WORK_SPREAD * WORK_STRIDE);
        CA_CUDA(cudaMemcpyAsync(w.data(), h->match_work, sizeof(unsigned long long) * w.size(),
                                cudaMemcpyDeviceToHost, h->stream));
        CA_CUDA(cudaStreamSynchronize(h->stream));
        unsigned long long s = 0;
        for (int i = 0; i < WORK_SPREAD; i++) s += w[(size_t)i * WORK_STRIDE];
        *rounds = (int32_t)s;
    }
    return CUALIGN_OK;
}

} // namespace cualign
