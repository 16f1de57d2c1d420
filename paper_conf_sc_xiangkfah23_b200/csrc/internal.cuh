// internal.cuh -- shared internals of libcualign_bp (CUDA, sm_100a).
// Not part of the ABI; the ABI is include/cualign_bp.h.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdarg.h>
#include <string>
#include <vector>

#include "../../include/cualign_bp.h"

#include <utility>

namespace cualign {

// ------------------------------------------------------------ probe knobs
// Measurement variants (timing probes, alternative launch shapes) are read
// from the environment ONLY in a probe build (-DCUALIGN_PROBES, see
// build.py --probes; never the product library): some of them skip work and
// give wrong results.  In the product build probe_knob() is the default.
#ifdef CUALIGN_PROBES
int probe_knob(const char *name, int dflt);
#else
inline int probe_knob(const char *, int dflt) { return dflt; }
#endif

// ------------------------------------------------------------------ errors
void set_error(const char *fmt, ...);
void clear_error();

#define CA_CUDA(call)                                                              \
    do {                                                                           \
        cudaError_t _e = (call);                                                   \
        if (_e != cudaSuccess) {                                                   \
            ::cualign::set_error("%s:%d: %s: %s", __FILE__, __LINE__, #call,       \
                                 cudaGetErrorString(_e));                          \
            return _e == cudaErrorMemoryAllocation ? CUALIGN_ENOMEM : CUALIGN_ECUDA; \
        }                                                                          \
    } while (0)

#define CA_TRY(call)                                  \
    do {                                              \
        cualign_status _s = (call);                   \
        if (_s != CUALIGN_OK) return _s;              \
    } while (0)

// ------------------------------------------------------------- L structure
// Device layout of the candidate graph L (row a1 of SURVEY §8):
//   La, Lb, w   canonical (a, b)-sorted edge list (edge id = index)
//   Arow        A-side rows: edges of A vertex a are Arow[a] .. Arow[a+1]-1
//   Bptr/Bedge  B-side incidence: Bedge[Bptr[b] .. Bptr[b+1]-1] = edge ids
//               of B vertex b, ascending
struct LDev {
    int32_t nA = 0, nB = 0;
    int64_t m = 0;
    int32_t *La = nullptr, *Lb = nullptr;
    double *w = nullptr;
    int64_t *Arow = nullptr, *Bptr = nullptr;
    int32_t *Bedge = nullptr;
};

// Device-side round bookkeeping (persistent across rounds: best).
// Mate arrays live in two slots of [2 instances][n_A] (cualign_bp::mates):
// a rounding writes slot wslot; if it improves the best, that slot becomes
// best_slot and the next rounding writes the other one -- the best matching is
// never copied (Alg. 2 l.22-24 keep bestM by reference).
struct RoundDev {
    unsigned int flag[2][2];      // [round parity][instance]: a match happened
    int rounds[2];
    unsigned long long overlap[2];
    unsigned long long card[2];
    double weight[2];
    double best_score;
    int best_iter;
    int improved;
    int source;
    unsigned int done;            // k_eval blocks finished (last-block final reduction)
    unsigned int gbar;            // k_eval<COLLECT>: blocks past the collect pass (grid barrier)
    int best_slot, best_source;   // where bestM lives: mates[best_slot][best_source] (valid if best_iter > 0)
    int wslot;                    // slot the next rounding writes (= 1 - best_slot)
    int last_slot;                // slot the last rounding wrote
    cualign_round_info info;
};

struct EventPair {
    cudaEvent_t a, b;
};

} // namespace cualign

struct cualign_bp {
    int dev = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    double alpha = 0, beta = 0, gamma = 1;
    uint32_t flags = 0;
    int num_sms = 148;

    cualign::LDev L;

    // sharding: this handle owns the L edges [e0, e1) -- whole
    // A rows [a0, a1) -- and the S rows of those edges.  world == 1: all.
    int32_t rank = 0, world = 1;
    int64_t e0 = 0, e1 = 0;
    int32_t a0 = 0, a1 = 0;
    std::vector<int64_t> bounds;         // world+1 edge boundaries (identical on all shards)
    int64_t s_total = 0, nsq_total = 0;  // global nnz(S), squares
    void *comm = nullptr;                // ncclComm_t of a process-sharded handle
    std::vector<cualign_bp *> vshards;   // in-process virtual shards (loopback group handle)
    double2 *Btop_part = nullptr;        // per-shard partial B-side top-2 (before the merge)
    double2 *Btop_all = nullptr;         // world x nB gathered partials
    int64_t *Bptr_loc = nullptr;         // B incidence of the owned edges (top-2 partials)
    int32_t *Bedge_loc = nullptr;
    // sharded square-pass halo (SURVEY §8(e) "S halo"): the squares {e < f}
    // of the owned rows touch f > e, i.e. edges of this or HIGHER shards only.
    // need: sorted remote f this shard reads u_f of and adds F_fe to, grouped
    // by owner (need_off[q]..need_off[q+1]); give: owned ids the lower shards
    // need, grouped by requester (give_off[r]..give_off[r+1])
    int32_t *halo_need = nullptr, *halo_give = nullptr;
    std::vector<int64_t> need_off, give_off;
    int64_t n_need = 0, n_give = 0;
    int64_t nsq_split = -1;            // sharded: squares [0, nsq_split) read owned f only (no halo);
                                       // [nsq_split, nsq) need the u halo (-1: no split)
    cudaStream_t cstream = nullptr;    // sharded: exchange stream (halo overlapped with the local squares)
    double *hu_out = nullptr, *hu_in = nullptr;                // packed u_f: give side -> need side
    unsigned long long *ht_out = nullptr, *ht_in = nullptr;    // packed F sums: need side -> give side

    // S: CSR over edge ids (rows [e0, e1)), and the square layout
    int64_t s = 0, nsq = 0, max_row = 0;
    int64_t *Srp = nullptr;      // (e1-e0)+1, indexed e - e0
    int32_t *Scol = nullptr;     // s
    int64_t *sq_rp = nullptr;    // (e1-e0)+1: row e has sq_rp[e-e0+1]-sq_rp[e-e0] squares {e<f} (build offsets)
    int2 *sq_ef = nullptr;       // nsq: (e, f), e < f, sorted by (e, f) inside (e block, f block) tiles
    int sq_tile_log = 0;         // tile blocks of 2^sq_tile_log edges (0: plain (e, f) order)
    double2 *sq_val = nullptr;   // nsq: (S^p_ef, S^p_fe)
    float2 *sq_val32 = nullptr;  // same, CUALIGN_FLAG_FP32_S storage (sq_val unused then)
    longlong2 *sq_pos = nullptr; // nsq: (pos(e,f), pos(f,e)) in the CSR; built lazily
    // packed square stream of the fast square pass (DESIGN.md "Packed square
    // indices"): word q = (e - eb) << SQP_FBITS | (f - fb) for the chunk's
    // (eb, fb); chunks of <= SQP_CHUNK consecutive squares, int4 (q0, n, eb, fb)
    uint32_t *sqp_w = nullptr;   // nsq (+4 padding)
    int4 *sqp_desc = nullptr;    // sqp_nchunks
    int64_t sqp_nchunks = 0;     // 0: packed stream not built (the int2 stream is used)
    int64_t sqp_split_chunk = 0; // first chunk at or after nsq_split (sharded square parts)

    // fixed-point accumulator of the F row sums (fast mode)
    int fp_bits = 0;
    double fp_scale = 1.0, fp_inv = 1.0;

    // per-edge state (Alg. 2 l.5, :158); d^p is never used (reading Z16)
    double *yc = nullptr, *zc = nullptr, *yp = nullptr, *zp = nullptr;
    double *d = nullptr, *u = nullptr;
    unsigned long long *tacc = nullptr; // fast mode: sum_f F_ef in fixed point
    double *texact = nullptr;           // exact mode: sum_f F_ef, oracle order
    double *Ffull = nullptr;            // exact mode: F in CSR order
    int64_t nchunks = 0;                // B incidence chunks (k_top2B load balance)
    int64_t *Bcp = nullptr;             // nB+1: chunks of B vertex b are Bcp[b]..Bcp[b+1]-1
    int4 *cdesc = nullptr;              // nchunks: (start, end, owning B vertex, first chunk of a hub or -1)
    double2 *Bct = nullptr;             // nchunks: (max1, max2) of z^p over the chunk
    unsigned int *Bcnt = nullptr;       // nB: chunks finished (hub columns' last-arriver merge)
    unsigned int *sq_ctr = nullptr;     // 2: square-pass chunk queue head, CTAs done (self-resetting)
    double2 *Atop = nullptr, *Btop = nullptr; // per-vertex (max1, max2) of y^p / z^p
    int64_t comm_calls = 0, comm_bytes_in = 0; // exchanges (sharded handles)
    double comm_ms = 0.0;
    std::vector<cualign::EventPair> comm_events;
    int32_t p = 0;                      // host mirror of the iteration count
    int *p_dev = nullptr;               // device iteration count (kernels read p_dev + 1)
    double2 *gh_dev = nullptr;          // gh[p] = (gamma^p, 1 - gamma^p)
    int64_t gh_cap = 0;

    // CUDA graphs of one step (iterate(1) [+ round]); [0] = no round, [1] = with round
    cudaStream_t gstream = nullptr;     // capture / replay stream (never the legacy stream)
    cudaStream_t gstream2 = nullptr;    // capture side branch: rounding overlapped with the square pass
    cudaStream_t gstream3 = nullptr;    // capture side branch: deferred evaluate
    cudaEvent_t eval_ev = nullptr;      // deferred evaluate done (the next collect waits for it)
    cudaEvent_t join3_ev = nullptr;     // gstream3 joins the graph's main stream
    bool defer_eval = false;            // pipelined graphs evaluate round k one step later
    cudaEvent_t sync_ev[2] = {nullptr, nullptr};
    cudaEvent_t fork_ev[2] = {nullptr, nullptr};
    bool capturing = false;
    int capture_what = 0;
    // graph slots: [0, 4) = CUALIGN_RUN_* bits (one step); PSLOT(kind, wb) =
    // the pipelined step graphs: kind 0 = iterate
    // into buffer wb, 1 = rounding of buffer 1-wb beside iterate into wb,
    // 2 = rounding of buffer wb
    static constexpr int NSLOT = 15;  // pipelined kinds 0-4 x 2 buffers (4..13) + SERIAL_SLOT (14)
    cudaGraphExec_t graph[2][NSLOT] = {};                   // [timed][slot]
    cudaGraphExec_t shard_graph = nullptr;                  // sharded: one iteration (all exchanges) as a graph
    struct StepCounts {
        int64_t launches = 0, class_launches[CUALIGN_NUM_KERNEL_CLASSES] = {}, comm_calls = 0, comm_bytes_in = 0;
    };
    std::vector<StepCounts> shard_step_counts;              // per shard: what one replay launches / exchanges
    bool shard_warm = false;                                // one eager sharded step done (NCCL connected)
    std::vector<const void *> shard_graph_gh;               // the shards' gamma tables the graph reads
    int64_t graph_launches[2][NSLOT] = {};                  // kernels per replay
    int64_t graph_class_launches[2][NSLOT][CUALIGN_NUM_KERNEL_CLASSES] = {};
    std::vector<std::pair<int, cualign::EventPair>> graph_events[NSLOT]; // timed graphs' event nodes
    // step pipeline: y^c, z^c double buffers ([0] = yc/zc, the current
    // iteration's outside a pipelined run), the iteration the rounding
    // kernels report (round_p; = p_dev except in a pipelined run)
    double *yc_b1 = nullptr, *zc_b1 = nullptr;
    int pipe_mode = -1;                 // step schedule: -1 undecided, 0 forked graph, 1 pipelined, 2 serial
    int sched_param = 0;                // cualign_params.schedule (0 = library's choice)
    int tile_log_param = 0;             // cualign_params.square_tile_log (0 = SQ_TILE_LOG, -1 = none)
    int top2_tg = 0;                    // k_top2 lanes per tile while capturing (0: default; pipelined graphs: 1)
    int sq_ctas = 0;                    // square-pass CTAs per SM while capturing (0: as many as fit)
    bool pipe_join_front = false;       // pipelined graphs: rounding joins before the square pass
    bool probe_no_eval = false;         // probe build timing probe: pipelined rounding without evaluate
    int *rp_dev = nullptr;
    const int *round_p = nullptr;

    // matching (two instances: y and z)
    int32_t *candA = nullptr, *candB = nullptr, *mateB = nullptr;
    int32_t *mates = nullptr; // [2 slots][2 instances][n_A]: matched edge per A vertex (RoundDev slots)
    int2 *mvA = nullptr;      // n_A: (M_y(i), M_z(i)) as B vertices (-1: unmatched), for evaluate
    unsigned long long *suit = nullptr; // Suitor slots, 2 instances x max(nA, nB)
    // sharded rounding (NEXT-1): replicated global suitors per (instance, B vertex)
    unsigned long long *dist_gx = nullptr, *dist_wxl = nullptr, *dist_wxg = nullptr, *dist_cnt = nullptr;
    int32_t *dist_gi = nullptr, *dist_wid = nullptr, *dist_hold = nullptr, *dist_act = nullptr;
    int dist_rounds = 0; // merge rounds of the last sharded rounding
    unsigned long long *dist_cnt_host = nullptr; // pinned: active count after each round of a batch
    double *partial_w = nullptr;
    int match_grid = 0, match_block = 256, eval_grid = 1, evalc_grid = 1;
    unsigned long long *match_work = nullptr; // proposals (suitor) or rounds, per instance
    int32_t *squeue = nullptr;                // Suitor rounds: queued proposers (3 buffers x NQ sub-queues of qcap)
    int *qcnt = nullptr;                      // sub-queue counters
    int64_t qcap = 0;
    int q2_grid = 1;                          // chain-form grid (one wave)
    int qr_grid = 1;                          // proposal-round grid (one wave)
    bool propose_from_b = false;              // suitor: proposing side (smaller max degree)
    // graphs A and B (CSR), kept for evaluate: overlap = #A edges {i,j} with
    // (M(i), M(j)) in E_B
    int64_t *Bp = nullptr;
    int32_t *Bj = nullptr;
    int2 *Apairs = nullptr;  // undirected A edges (i, j), i < j
    unsigned long long *Bhash = nullptr; // E_B membership: open-addressing set of (u << 32 | v), u < v
    int Bhash_log = 0;                   // 2^Bhash_log slots (load <= 1/2)
    int64_t nApairs = 0;
    int64_t max_deg_a = 0, max_deg_b = 0;     // max degree of A / B vertices in L
    cualign::RoundDev *rd = nullptr;
    cualign_round_info last_info{};
    bool have_info = false;

    // diagnostics
    bool timing = false;
    int64_t launches = 0;
    int64_t class_launches[CUALIGN_NUM_KERNEL_CLASSES] = {};
    std::vector<cualign::EventPair> events[CUALIGN_NUM_KERNEL_CLASSES];
    std::vector<cudaEvent_t> event_pool;
    double class_ms[CUALIGN_NUM_KERNEL_CLASSES] = {};

    std::vector<std::pair<void *, size_t>> allocs;
    int64_t device_bytes = 0;
};

namespace cualign {

// ---------------------------------------------- programmatic dependent launch
// Kernels of the step chain start with pdl_wait(): launched with
// launch_pdl they are scheduled while their predecessor drains (its launch
// latency hidden); the wait returns once the predecessor grid has completed
// and its memory is visible.  Launched normally, the wait is a no-op.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args &&...args)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// --------------------------------------------------------------- memory
cualign_status dmalloc(cualign_bp *h, void **p, size_t bytes);
cudaMemPool_t temp_pool(int dev); // cached pool for init temporaries (nullptr: use the default)

// init temporaries: stream-ordered from a cached pool of their own (no
// device-wide synchronisation in cudaFree, memory reused across handles)
struct TmpBuf {
    void *p = nullptr;
    cudaStream_t s = nullptr;
    ~TmpBuf()
    {
        if (p) cudaFreeAsync(p, s);
    }
};
inline cudaError_t tmalloc(cualign_bp *h, TmpBuf &b, size_t bytes)
{
    b.s = h->stream;
    cudaMemPool_t pool = temp_pool(h->dev);
    if (pool) return cudaMallocFromPoolAsync(&b.p, bytes ? bytes : 1, pool, h->stream);
    return cudaMallocAsync(&b.p, bytes ? bytes : 1, h->stream);
}
template <class T>
inline cualign_status dalloc(cualign_bp *h, T **p, size_t n)
{
    return dmalloc(h, reinterpret_cast<void **>(p), n * sizeof(T));
}
void dfree(cualign_bp *h, void *p);
void dfree_all(cualign_bp *h);

// ------------------------------------------------- B-edge membership set
// Evaluate asks "is (M(i), M(j)) an edge of B?" once per
// undirected A edge and matching.  A sorted-row binary search is ~5 dependent
// loads; this set answers in ~1: key (min << 32 | max), multiplicative hash,
// linear probing, empty = ~0.
constexpr unsigned long long BHASH_EMPTY = ~0ull;
__host__ __device__ __forceinline__ unsigned long long bhash_key(int32_t u, int32_t v)
{
    const uint32_t lo = (uint32_t)(u < v ? u : v), hi = (uint32_t)(u < v ? v : u);
    return ((unsigned long long)lo << 32) | hi;
}
__host__ __device__ __forceinline__ uint64_t bhash_slot(unsigned long long key, int log2n)
{
    return (key * 0x9E3779B97F4A7C15ull) >> (64 - log2n);
}
__device__ __forceinline__ bool bhash_has(const unsigned long long *__restrict__ T, int log2n, unsigned long long key)
{
    const uint64_t mask = (1ull << log2n) - 1;
    for (uint64_t i = bhash_slot(key, log2n);; i = (i + 1) & mask) {
        const unsigned long long x = __ldg(T + i);
        if (x == key) return true;
        if (x == BHASH_EMPTY) return false;
    }
}

// ------------------------------------------------------------ diagnostics
// CUALIGN_INIT_TRACE=1: synchronise and print the time of each init phase
void init_trace(cualign_bp *h, const char *what);

// ------------------------------------------------------- launch accounting
// an exchange between shards (NCCL or loopback copies): bytes received by
// the shard and, with timing on, its event time (not counted as a launch)
struct CommScope {
    cualign_bp *h;
    cudaEvent_t b = nullptr;
    CommScope(cualign_bp *h_, int64_t bytes_in);
    ~CommScope();
};

struct KScope {
    cualign_bp *h;
    int cls;
    cudaEvent_t b = nullptr;
    KScope(cualign_bp *h_, int cls_);
    ~KScope();
};

// ------------------------------------------------------------ subsystems
// init.cu
cualign_status build_L(cualign_bp *h, LDev &L, const cualign_edges *E, bool device_ptrs,
                       bool validate, int32_t nA, int32_t nB);
cualign_status upload_graph(cualign_bp *h, const cualign_graph *g, const char *what, int64_t **rp, int32_t **col,
                            int64_t *nnz_out); // copy + validate (Z14); device CSR owned by h
cualign_status build_problem(cualign_bp *h, const cualign_graph *A, const cualign_graph *B,
                             const cualign_edges *E);
cualign_status ensure_sq_pos(cualign_bp *h);
cualign_status ensure_csr(cualign_bp *h);
cualign_status tile_squares(cualign_bp *h);
constexpr int SQ_TILE_LOG = 21; // square tiles: blocks of 2^21 edges (2 x 32 MB of u + tacc per tile)
cualign_status pack_squares(cualign_bp *h); // packed square stream from sq_ef (after every reorder)
constexpr int EVAL_BS = 128;                // k_eval block size (match.cu)
constexpr int SQP_CHUNK = 512;              // squares per packed chunk (= square-pass stage)
constexpr int SQP_FBITS = 21;               // f - fb in the low bits (f blocks of 2^21 = the tile blocks)
constexpr int SQP_EBITS = 32 - SQP_FBITS;   // e - eb in the high bits

// api.cu
void invalidate_graphs(cualign_bp *h);

// bp.cu
cualign_status ensure_gh(cualign_bp *h, int64_t pmax); // gamma^p table covers p <= pmax
cualign_status bp_setup(cualign_bp *h);                // B chunks
cualign_status bp_fsum(cualign_bp *h);                 // t <- sum_f F(S^p) (init / set_state)
cualign_status bp_iterate(cualign_bp *h, int32_t n);   // Alg. 2 l.9-16, n times
cualign_status bp_iterate_front(cualign_bp *h);        // advance p, top-2, k_edge
cualign_status bp_iterate_back(cualign_bp *h);         // square pass
cualign_status bp_iterate_back_range(cualign_bp *h, int64_t q0, int64_t q1); // square pass over [q0, q1)
cualign_status bp_top2(cualign_bp *h);                 // per-vertex top-2 of the current y^p, z^p
cualign_status bp_front_top2(cualign_bp *h);           // advance p, top-2 (partial B when sharded)
cualign_status bp_front_edge(cualign_bp *h);           // k_edge on the owned edges
cualign_status bp_merge_top2(cualign_bp *h);           // gathered B partials -> Btop
cualign_status bp_add_u64(cualign_bp *h, unsigned long long *dst, const unsigned long long *src, int64_t n);

// shard.cu
cualign_status shard_setup(cualign_bp *h);  // square-pass halo lists (after the S build)
cualign_status shard_fsum(cualign_bp *h);
cualign_status shard_iterate(cualign_bp *h, int32_t n);
cualign_status shard_round(cualign_bp *h);
cualign_status nccl_init_comm(cualign_bp *h, const void *unique_id);
void nccl_free_comm(cualign_bp *h);
cualign_status nccl_unique_id(void *out, int32_t len);
cualign_status bp_sample_squares(cualign_bp *h, const int32_t *edges, int64_t n, int64_t cap, int32_t *e_out,
                                 int32_t *f_out, double *v_ef, double *v_fe, int64_t *n_out);
cualign_status bp_scatter_Sp(cualign_bp *h, double *Sfull_dev);        // squares -> CSR
cualign_status bp_gather_Sp(cualign_bp *h, const double *Sfull_dev);   // CSR -> squares

// match.cu
cualign_status quality_eval(cualign_bp *h, const cualign_graph *A, const cualign_graph *B, const int32_t *map_ab,
                            const int32_t *truth, cualign_quality *out); // NEXT-4 (quality.cu)
cualign_status knn_build(cualign_bp *h, const float *YA, int32_t n_a, const float *YB, int32_t n_b, int32_t d,
                         int32_t k, int32_t *La, int32_t *Lb, double *Lw); // NEXT-2 (knn.cu)
cualign_status match_setup(cualign_bp *h);
cualign_status match_round(cualign_bp *h);  // a7 + a8 on the device
cualign_status match_round_deferred(cualign_bp *h, int set, cudaEvent_t before_collect); // a7 (pipelined)
cualign_status eval_round_deferred(cualign_bp *h, int set);                              // a8, one step later
bool can_defer_eval(const cualign_bp *h);
cualign_status match_evaluate(cualign_bp *h); // a8 on the round's mate slot (collect done)
// sharded rounding (NEXT-1), driven by shard_round: begin, then rounds of
// local -> all-reduce MAX(dist_wxg) -> cand -> all-reduce MIN(dist_wid) ->
// update -> all-reduce SUM(dist_cnt) until the count is 0, then finish
cualign_status dist_match_begin(cualign_bp *h);
cualign_status dist_match_local(cualign_bp *h);
cualign_status dist_match_cand(cualign_bp *h);
cualign_status dist_match_update(cualign_bp *h);
cualign_status dist_match_finish(cualign_bp *h);
cualign_status match_standalone(cualign_bp *h, const double *x_dev, int32_t *rounds);

// helpers
inline int grid_for(int64_t n, int block, int max_blocks)
{
    int64_t g = (n + block - 1) / block;
    if (g < 1) g = 1;
    if (g > max_blocks) g = max_blocks;
    return (int)g;
}

} // namespace cualign
