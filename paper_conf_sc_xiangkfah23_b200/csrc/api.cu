// api.cu -- the C ABI (include/cualign_bp.h): argument checks, handle
// lifetime, state transfer, diagnostics.  All compute is in init.cu, bp.cu,
// match.cu.
#include "internal.cuh"

#include <mutex>

#include <chrono>

#include <math.h>
#include <string.h>

namespace cualign {

static thread_local char g_err[1024] = "";

#ifdef CUALIGN_PROBES
int probe_knob(const char *name, int dflt)
{
    const char *v = getenv(name);
    return v ? atoi(v) : dflt;
}
#endif

void set_error(const char *fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

void clear_error() { g_err[0] = 0; }

// Device memory comes from the device's stream-ordered pool with an unlimited
// release threshold: freed blocks stay cached in the process, so a new handle
// (a new alignment) reuses them instead of paying cudaMalloc / cudaFree.
static void keep_pool(int dev)
{
    static bool done[64] = {};
    if (dev < 0 || dev >= 64 || done[dev]) return;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    (void)cudaGetLastError();
    done[dev] = true;
}

// Init temporaries (sort buffers, counts) come from a second pool, also
// cached: taken from the main pool they would leave holes between the
// handle's persistent arrays, and the next handle's persistent allocations
// would then grow the main pool (measured: alloc_state 1.5 -> 240 ms).
cudaMemPool_t temp_pool(int dev)
{
    static cudaMemPool_t pools[64] = {};
    static bool made[64] = {};
    static std::mutex mu; // handles may be created from several host threads
    if (dev < 0 || dev >= 64) return nullptr;
    std::lock_guard<std::mutex> lock(mu);
    if (!made[dev]) {
        made[dev] = true;
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        if (cudaMemPoolCreate(&pools[dev], &props) == cudaSuccess) {
            uint64_t thr = UINT64_MAX;
            cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &thr);
        } else {
            pools[dev] = nullptr;
        }
        (void)cudaGetLastError();
    }
    return pools[dev];
}

cualign_status dmalloc(cualign_bp *h, void **p, size_t bytes)
{
    if (bytes == 0) bytes = 16;
    keep_pool(h->dev);
    cudaError_t e = cudaMallocAsync(p, bytes, h->stream);
    if (e != cudaSuccess) {
        *p = nullptr;
        set_error("cudaMalloc(%zu bytes) failed: %s", bytes, cudaGetErrorString(e));
        (void)cudaGetLastError();
        return e == cudaErrorMemoryAllocation ? CUALIGN_ENOMEM : CUALIGN_ECUDA;
    }
    h->allocs.push_back({*p, bytes});
    h->device_bytes += (int64_t)bytes;
    return CUALIGN_OK;
}

void dfree(cualign_bp *h, void *p)
{
    for (auto &a : h->allocs)
        if (a.first == p && p) {
            cudaFreeAsync(p, h->stream);
            h->device_bytes -= (int64_t)a.second;
            a.first = nullptr;
            a.second = 0;
        }
}

void dfree_all(cualign_bp *h)
{
    for (auto &a : h->allocs)
        if (a.first) cudaFreeAsync(a.first, h->stream);
    cudaStreamSynchronize(h->stream);
    h->allocs.clear();
    h->device_bytes = 0;
}

static cudaEvent_t get_event(cualign_bp *h)
{
    if (!h->event_pool.empty()) {
        cudaEvent_t e = h->event_pool.back();
        h->event_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}

// While a graph is being captured, timing events become event-record nodes
// (cudaEventRecordExternal) owned by the graph; they are read after each replay.
KScope::KScope(cualign_bp *h_, int cls_) : h(h_), cls(cls_)
{
    if (h->timing) {
        b = get_event(h);
        if (h->capturing) cudaEventRecordWithFlags(b, h->stream, cudaEventRecordExternal);
        else cudaEventRecord(b, h->stream);
    }
}

KScope::~KScope()
{
    h->launches++;
    h->class_launches[cls]++;
    if (h->timing && b) {
        cudaEvent_t e = get_event(h);
        if (h->capturing) {
            cudaEventRecordWithFlags(e, h->stream, cudaEventRecordExternal);
            h->graph_events[h->capture_what].push_back({cls, {b, e}});
        } else {
            cudaEventRecord(e, h->stream);
            h->events[cls].push_back({b, e});
        }
    }
}

CommScope::CommScope(cualign_bp *h_, int64_t bytes_in) : h(h_)
{
    h->comm_calls++;
    h->comm_bytes_in += bytes_in;
    if (h->timing && !h->capturing) {
        b = get_event(h);
        cudaEventRecord(b, h->stream);
    }
}

CommScope::~CommScope()
{
    if (b) {
        cudaEvent_t e = get_event(h);
        cudaEventRecord(e, h->stream);
        h->comm_events.push_back({b, e});
    }
}

void invalidate_graphs(cualign_bp *h)
{
    if (h->shard_graph) {
        cudaGraphExecDestroy(h->shard_graph);
        h->shard_graph = nullptr;
    }
    for (int t = 0; t < 2; t++)
        for (int r = 0; r < cualign_bp::NSLOT; r++)
            if (h->graph[t][r]) {
                cudaGraphExecDestroy(h->graph[t][r]);
                h->graph[t][r] = nullptr;
            }
    for (int r = 0; r < cualign_bp::NSLOT; r++) {
        for (auto &pe : h->graph_events[r]) {
            h->event_pool.push_back(pe.second.a);
            h->event_pool.push_back(pe.second.b);
        }
        h->graph_events[r].clear();
    }
}

__global__ void k_copy_int(int *dst, const int *src) { *dst = *src; }
__global__ void k_incr_int(int *x) { *x += 1; }

static inline int pslot(int kind, int wb) { return 4 + 2 * kind + wb; }
static constexpr int SERIAL_SLOT = 14; // one step as ONE graph: iterate(1), then the rounding (no fork)

// The pipelined graphs' work (see capture_step): the y^c / z^c buffers are
// selected by pointing h->yc / h->zc at them while the kernels are captured.
static cualign_status capture_pipelined(cualign_bp *h, int kind, int wb)
{
    // k_top2 lanes per tile in the pipelined graphs.  Round 1 (the rounding
    // then ran ~0.23 ms beside it) took 1 lane: 4x fewer threads left SM
    // slots to the rounding.  Round 2 (packed square stream, 3 proposal
    // rounds) measured the bench window on O: 1 lane 1421-1440 it/s, 2 lanes
    // 1449-1469, 4 lanes 1465 -- 2 lanes, as in the serial graph.
    struct TgScope {
        cualign_bp *h;
        ~TgScope() { h->top2_tg = 0; h->sq_ctas = 0; h->probe_no_eval = false; }
    } tg_scope{h};
    h->top2_tg = probe_knob("CUALIGN_PIPE_TOP2_TG", 2);
    // the square pass leaves SM room to the rounding running beside it
    static const int pipe_sq = probe_knob("CUALIGN_PIPE_SQ_CTAS", 0);
    h->sq_ctas = pipe_sq;
    h->pipe_join_front = probe_knob("CUALIGN_PIPE_JOIN_FRONT", 0) != 0;
    h->probe_no_eval = probe_knob("CUALIGN_PIPE_NO_EVAL", 0) != 0;
    double *yc0 = h->yc, *zc0 = h->zc;
    double *yb[2] = {yc0, h->yc_b1}, *zb[2] = {zc0, h->zc_b1};
    cualign_status st = CUALIGN_OK;
    auto round_of = [&](int buf) -> cualign_status {
        // the rounding reports its own iteration counter (rp = iteration
        // rounded), advanced at the start of every pipelined rounding
        {
            KScope ks(h, CUALIGN_K_OTHER);
            k_incr_int<<<1, 1, 0, h->stream>>>(h->rp_dev);
            CA_CUDA(cudaGetLastError());
        }
        h->yc = yb[buf];
        h->zc = zb[buf];
        h->round_p = h->rp_dev;
        cualign_status r = match_round(h);
        h->round_p = nullptr;
        return r;
    };
    if (kind == 0) {
        {
            KScope ks(h, CUALIGN_K_OTHER);
            k_copy_int<<<1, 1, 0, h->stream>>>(h->rp_dev, h->p_dev); // rounds done so far = p
            if (cudaGetLastError() != cudaSuccess) st = CUALIGN_ECUDA;
        }
        h->yc = yb[wb];
        h->zc = zb[wb];
        if (st == CUALIGN_OK) st = bp_iterate(h, 1);
    } else if (h->defer_eval && kind != 0) {
        // deferred evaluate: a round's
        // matching beside the next iteration, its evaluate one graph later
        // beside the iteration after that; the matching's collect pass waits
        // for the previous round's evaluate.  The proposal counters and y^c /
        // z^c of a round use set = buffer = wb of the iteration it rounds.
        //   kind 1: iteration p || match(p-1)                     (p = 2)
        //   kind 3: iteration p || match(p-1) || eval(p-2)        (p >= 3)
        //   kind 4: eval(n-1)                                     (drain, n >= 2)
        //   kind 2: match(n), eval(n)                             (drain)
        auto eval_of = [&](int set) -> cualign_status {
            {
                KScope ks(h, CUALIGN_K_OTHER);
                k_incr_int<<<1, 1, 0, h->stream>>>(h->rp_dev);
                CA_CUDA(cudaGetLastError());
            }
            h->round_p = h->rp_dev;
            cualign_status r = eval_round_deferred(h, set);
            h->round_p = nullptr;
            return r;
        };
        auto match_of = [&](int buf, cudaEvent_t ev) -> cualign_status {
            h->yc = yb[buf];
            h->zc = zb[buf];
            return match_round_deferred(h, buf, ev);
        };
        if (kind == 2) {
            st = match_of(wb, nullptr);
            if (st == CUALIGN_OK) st = eval_of(wb);
        } else if (kind == 4) {
            st = eval_of(wb);
        } else {
            const bool with_eval = kind == 3;
            // the evaluate runs on the iteration's stream ahead of its k_edge,
            // beside the matching's first proposals (bench window on O: 1506-
            // 1511 it/s; on a third stream beside k_edge: 1492-1494; evaluate
            // in the round's own graph: 1469).  Probe build:
            // CUALIGN_PIPE_EVAL_MAIN=0 takes the third stream.
            static const bool eval_main = probe_knob("CUALIGN_PIPE_EVAL_MAIN", 1) != 0;
            // probe build: CUALIGN_PIPE_EVAL_LATE=1 starts the evaluate on the
            // third stream after k_top2, beside the square pass
            static const bool eval_late = probe_knob("CUALIGN_PIPE_EVAL_LATE", 0) != 0;
            cudaStream_t es = (eval_main && !eval_late) ? h->gstream : h->gstream3;
            if (cudaEventRecord(h->fork_ev[0], h->gstream) != cudaSuccess ||
                cudaStreamWaitEvent(h->gstream2, h->fork_ev[0], 0) != cudaSuccess ||
                (with_eval && !eval_main && !eval_late &&
                 cudaStreamWaitEvent(h->gstream3, h->fork_ev[0], 0) != cudaSuccess))
                st = CUALIGN_ECUDA;
            if (st == CUALIGN_OK && with_eval && eval_late) {
                // iteration front first; the evaluate forks after k_top2
                h->yc = yb[wb];
                h->zc = zb[wb];
                st = bp_iterate_front(h);
                if (st == CUALIGN_OK && (cudaEventRecord(h->join3_ev, h->gstream) != cudaSuccess ||
                                         cudaStreamWaitEvent(h->gstream3, h->join3_ev, 0) != cudaSuccess))
                    st = CUALIGN_ECUDA;
            }
            if (st == CUALIGN_OK && with_eval) {
                h->stream = es;
                st = eval_of(wb); // round p-2 read buffer wb
                if (st == CUALIGN_OK && cudaEventRecord(h->eval_ev, es) != cudaSuccess) st = CUALIGN_ECUDA;
                h->stream = h->gstream;
            }
            if (st == CUALIGN_OK) {
                h->stream = h->gstream2;
                st = match_of(1 - wb, with_eval ? h->eval_ev : nullptr);
                h->stream = h->gstream;
            }
            h->yc = yb[wb];
            h->zc = zb[wb];
            if (st == CUALIGN_OK && with_eval && eval_late) {
                st = bp_iterate_back(h);
                if (st == CUALIGN_OK) h->p += 1;
            } else if (st == CUALIGN_OK) {
                st = bp_iterate(h, 1);
            }
            if (st == CUALIGN_OK && (cudaEventRecord(h->fork_ev[1], h->gstream2) != cudaSuccess ||
                                     cudaStreamWaitEvent(h->gstream, h->fork_ev[1], 0) != cudaSuccess))
                st = CUALIGN_ECUDA;
            if (st == CUALIGN_OK && with_eval && (!eval_main || eval_late) &&
                (cudaEventRecord(h->join3_ev, h->gstream3) != cudaSuccess ||
                 cudaStreamWaitEvent(h->gstream, h->join3_ev, 0) != cudaSuccess))
                st = CUALIGN_ECUDA;
        }
    } else if (kind == 1) {
        // fork: the rounding of iteration p-1 (buffer 1-wb) beside all of
        // iteration p (writes buffer wb); the rounding reads only y^c, z^c of
        // p-1, w and L, which iteration p does not touch
        if (cudaEventRecord(h->fork_ev[0], h->gstream) != cudaSuccess ||
            cudaStreamWaitEvent(h->gstream2, h->fork_ev[0], 0) != cudaSuccess)
            st = CUALIGN_ECUDA;
        if (st == CUALIGN_OK) {
            h->stream = h->gstream2;
            st = round_of(1 - wb);
            h->stream = h->gstream;
        }
        h->yc = yb[wb];
        h->zc = zb[wb];
        // the join before the square pass (h->pipe_join_front): the rounding
        // overlaps only the latency-bound front (k_edge, k_top2) of iteration
        // p; the square pass, which needs every SM at full occupancy, runs alone
        if (h->pipe_join_front) {
            if (st == CUALIGN_OK) st = bp_iterate_front(h);
            if (st == CUALIGN_OK && (cudaEventRecord(h->fork_ev[1], h->gstream2) != cudaSuccess ||
                                     cudaStreamWaitEvent(h->gstream, h->fork_ev[1], 0) != cudaSuccess))
                st = CUALIGN_ECUDA;
            if (st == CUALIGN_OK) st = bp_iterate_back(h);
            if (st == CUALIGN_OK) h->p += 1;
        } else {
            if (st == CUALIGN_OK) st = bp_iterate(h, 1);
            if (st == CUALIGN_OK && (cudaEventRecord(h->fork_ev[1], h->gstream2) != cudaSuccess ||
                                     cudaStreamWaitEvent(h->gstream, h->fork_ev[1], 0) != cudaSuccess))
                st = CUALIGN_ECUDA;
        }
    } else {
        st = round_of(wb);
    }
    h->yc = yc0;
    h->zc = zc0;
    return st;
}

// Capture one step (iterate(1) [+ round]) on the handle's capture stream.
// slot < 4: what bits (bit 0 = iterate(1), bit 1 = round, CUALIGN_RUN_*);
// slot >= 4: a pipelined graph (pslot(kind, wb)).
static cualign_status capture_step(cualign_bp *h, int timed, int slot)
{
    const int what = slot < 4 ? slot : 0;
    const int32_t p_save = h->p;
    const int64_t l0 = h->launches;
    int64_t c0[CUALIGN_NUM_KERNEL_CLASSES];
    for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) c0[c] = h->class_launches[c];
    const bool timing_save = h->timing;
    cudaStream_t user = h->stream;
    h->timing = timed != 0;
    h->stream = h->gstream;
    h->capturing = true;
    h->capture_what = slot;
    cualign_status st = CUALIGN_OK;
    cudaError_t e = cudaStreamBeginCapture(h->gstream, cudaStreamCaptureModeThreadLocal);
    if (e == cudaSuccess) {
        if (slot == SERIAL_SLOT) {
            st = bp_iterate(h, 1);
            if (st == CUALIGN_OK) st = match_round(h);
        } else if (slot >= 4) {
            st = capture_pipelined(h, (slot - 4) / 2, (slot - 4) % 2);
        } else if (what == (CUALIGN_RUN_ITERATE | CUALIGN_RUN_ROUND)) {
            // the rounding of iteration p reads only y^c, z^c (or y^p, z^p),
            // w and L -- final after the first half -- and the square pass
            // touches none of them: fork the rounding onto a side branch so
            // the latency-bound matching overlaps the bandwidth-bound pass.
            st = bp_iterate_front(h);
            if (st == CUALIGN_OK && cudaEventRecord(h->fork_ev[0], h->gstream) != cudaSuccess) st = CUALIGN_ECUDA;
            if (st == CUALIGN_OK && cudaStreamWaitEvent(h->gstream2, h->fork_ev[0], 0) != cudaSuccess)
                st = CUALIGN_ECUDA;
            if (st == CUALIGN_OK) {
                h->stream = h->gstream2;
                st = match_round(h);
                h->stream = h->gstream;
            }
            if (st == CUALIGN_OK) st = bp_iterate_back(h);
            if (st == CUALIGN_OK && cudaEventRecord(h->fork_ev[1], h->gstream2) != cudaSuccess) st = CUALIGN_ECUDA;
            if (st == CUALIGN_OK && cudaStreamWaitEvent(h->gstream, h->fork_ev[1], 0) != cudaSuccess)
                st = CUALIGN_ECUDA;
            if (st == CUALIGN_OK) h->p += 1;
        } else {
            if (what & CUALIGN_RUN_ITERATE) st = bp_iterate(h, 1);
            if (st == CUALIGN_OK && (what & CUALIGN_RUN_ROUND)) st = match_round(h);
        }
        cudaGraph_t g = nullptr;
        cudaError_t e2 = cudaStreamEndCapture(h->gstream, &g);
        if (st == CUALIGN_OK && e2 != cudaSuccess) {
            set_error("graph capture: %s", cudaGetErrorString(e2));
            st = CUALIGN_ECUDA;
        }
        if (st == CUALIGN_OK) {
            e2 = cudaGraphInstantiate(&h->graph[timed][slot], g, 0);
            if (e2 != cudaSuccess) {
                set_error("graph instantiate: %s", cudaGetErrorString(e2));
                st = CUALIGN_ECUDA;
            }
        }
        if (g) cudaGraphDestroy(g);
    } else {
        set_error("graph capture: %s", cudaGetErrorString(e));
        st = CUALIGN_ECUDA;
    }
    h->capturing = false;
    h->stream = user;
    h->timing = timing_save;
    h->p = p_save;
    h->graph_launches[timed][slot] = h->launches - l0;
    for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) {
        h->graph_class_launches[timed][slot][c] = h->class_launches[c] - c0[c];
        h->class_launches[c] = c0[c];
    }
    h->launches = l0;
    (void)cudaGetLastError();
    return st;
}

// n steps through the captured graph; the user stream and the capture stream
// are ordered with events, so the caller's stream semantics are preserved.
static cualign_status run_graph(cualign_bp *h, int32_t n, int what)
{
    const int timed = h->timing ? 1 : 0;
    CA_TRY(ensure_gh(h, (int64_t)h->p + n + 1));
    if (!h->graph[timed][what]) CA_TRY(capture_step(h, timed, what));
    cudaGraphExec_t ge = h->graph[timed][what];
    CA_CUDA(cudaEventRecord(h->sync_ev[0], h->stream));
    CA_CUDA(cudaStreamWaitEvent(h->gstream, h->sync_ev[0], 0));
    for (int32_t k = 0; k < n; k++) {
        CA_CUDA(cudaGraphLaunch(ge, h->gstream));
        if (what & CUALIGN_RUN_ITERATE) h->p += 1;
        h->launches += h->graph_launches[timed][what];
        for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++)
            h->class_launches[c] += h->graph_class_launches[timed][what][c];
        if (timed) {
            CA_CUDA(cudaStreamSynchronize(h->gstream));
            for (auto &pe : h->graph_events[what]) {
                float ms = 0.f;
                if (cudaEventElapsedTime(&ms, pe.second.a, pe.second.b) == cudaSuccess) h->class_ms[pe.first] += ms;
            }
        }
    }
    if (what & CUALIGN_RUN_ROUND) h->have_info = true;
    CA_CUDA(cudaEventRecord(h->sync_ev[1], h->gstream));
    CA_CUDA(cudaStreamWaitEvent(h->stream, h->sync_ev[1], 0));
    return CUALIGN_OK;
}

void init_trace(cualign_bp *h, const char *what)
{
    static const bool on = probe_knob("CUALIGN_INIT_TRACE", 0) != 0;
    if (!on) return;
    static thread_local std::chrono::steady_clock::time_point t0;
    cudaStreamSynchronize(h->stream);
    const auto now = std::chrono::steady_clock::now();
    if (what[0] == '^') t0 = now;
    fprintf(stderr, "[init] %-24s %9.3f ms\n", what,
            std::chrono::duration<double, std::milli>(now - t0).count());
}

// second y^c / z^c buffers and the rounding's iteration counter of the step
// pipeline; allocated at init next to the first ones (a later allocation
// fragments the stream-ordered pool the next handle reuses)
static cualign_status alloc_pipeline(cualign_bp *h)
{
    CA_TRY(dalloc(h, &h->yc_b1, (size_t)h->L.m + 1));
    CA_TRY(dalloc(h, &h->zc_b1, (size_t)h->L.m + 1));
    CA_TRY(dalloc(h, &h->rp_dev, 1));
    return CUALIGN_OK;
}

// Launch graph slot `slot` once on the capture stream (capturing it first).
static cualign_status launch_slot(cualign_bp *h, int slot)
{
    const int timed = h->timing ? 1 : 0;
    if (!h->graph[timed][slot]) CA_TRY(capture_step(h, timed, slot));
    CA_CUDA(cudaGraphLaunch(h->graph[timed][slot], h->gstream));
    h->launches += h->graph_launches[timed][slot];
    for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) h->class_launches[c] += h->graph_class_launches[timed][slot][c];
    if (timed) {
        CA_CUDA(cudaStreamSynchronize(h->gstream));
        for (auto &pe : h->graph_events[slot]) {
            float ms = 0.f;
            if (cudaEventElapsedTime(&ms, pe.second.a, pe.second.b) == cudaSuccess) h->class_ms[pe.first] += ms;
        }
    }
    return CUALIGN_OK;
}

// Step pipeline: n x (iterate + round) where the
// rounding of iteration k runs beside iteration k+1.  Iteration k writes y^c,
// z^c into buffer wb_k = (n - k) & 1, so the rounding of k (next graph)
// reads the buffer iteration k+1 does not write, and the last iteration's
// values end in buffer 0 (h->yc, h->zc), as after an unpipelined run.
static cualign_status run_pipelined(cualign_bp *h, int32_t n, RoundDev *trace = nullptr)
{
    if (n <= 0) return CUALIGN_OK;
    CA_TRY(ensure_gh(h, (int64_t)h->p + n + 1));
    if (!h->yc_b1) CA_TRY(alloc_pipeline(h));
    CA_CUDA(cudaEventRecord(h->sync_ev[0], h->stream));
    CA_CUDA(cudaStreamWaitEvent(h->gstream, h->sync_ev[0], 0));
    const bool dfr = h->defer_eval;
    for (int32_t k = 1; k <= n; k++) {
        const int wb = (n - k) & 1;
        CA_TRY(launch_slot(h, pslot(k == 1 ? 0 : ((dfr && k >= 3) ? 3 : 1), wb)));
        h->p += 1;
        // the rounding (deferred: the evaluate) of iteration k-1 (k-2)
        // finished inside this graph: its result to the host, stream-ordered
        // before the next graph rewrites it
        const int r = dfr ? k - 3 : k - 2;
        if (trace && r >= 0)
            CA_CUDA(cudaMemcpyAsync(trace + r, h->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, h->gstream));
    }
    if (dfr && n >= 2) {
        CA_TRY(launch_slot(h, pslot(4, 1))); // evaluate of round n-1 (it read buffer 1)
        if (trace) CA_CUDA(cudaMemcpyAsync(trace + (n - 2), h->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, h->gstream));
    }
    CA_TRY(launch_slot(h, pslot(2, 0)));
    if (trace) CA_CUDA(cudaMemcpyAsync(trace + (n - 1), h->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, h->gstream));
    h->have_info = true;
    CA_CUDA(cudaEventRecord(h->sync_ev[1], h->gstream));
    CA_CUDA(cudaStreamWaitEvent(h->stream, h->sync_ev[1], 0));
    return CUALIGN_OK;
}

static void resolve_events(cualign_bp *h)
{
    for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) {
        for (auto &ep : h->events[c]) {
            float ms = 0.f;
            if (cudaEventSynchronize(ep.b) == cudaSuccess && cudaEventElapsedTime(&ms, ep.a, ep.b) == cudaSuccess)
                h->class_ms[c] += ms;
            h->event_pool.push_back(ep.a);
            h->event_pool.push_back(ep.b);
        }
        h->events[c].clear();
    }
    (void)cudaGetLastError();
}

static cualign_status check_params(const cualign_params *p)
{
    if (!p) {
        set_error("params is NULL");
        return CUALIGN_EINVAL;
    }
    if (!(p->alpha >= 0.0) || !isfinite(p->alpha)) {
        set_error("alpha must be finite and >= 0 (PAPER.md:64), got %g", p->alpha);
        return CUALIGN_EINVAL;
    }
    if (!(p->beta >= 0.0) || !isfinite(p->beta)) {
        set_error("beta must be finite and >= 0 (PAPER.md:64), got %g", p->beta);
        return CUALIGN_EINVAL;
    }
    if (!(p->gamma > 0.0 && p->gamma <= 1.0)) {
        set_error("gamma must be in (0, 1], got %g", p->gamma);
        return CUALIGN_EINVAL;
    }
    if (p->schedule < 0 || p->schedule > 3) {
        set_error("schedule must be 0 (automatic), 1 (pipelined), 2 (serial) or 3 (forked), got %d", p->schedule);
        return CUALIGN_EINVAL;
    }
    if (p->square_tile_log < -1 || p->square_tile_log > 30) {
        set_error("square_tile_log must be -1 (no tiles), 0 (automatic) or 1..30, got %d", p->square_tile_log);
        return CUALIGN_EINVAL;
    }
    if ((p->flags & CUALIGN_FLAG_FP32_S) && (p->flags & CUALIGN_FLAG_EXACT)) {
        set_error("CUALIGN_FLAG_FP32_S and CUALIGN_FLAG_EXACT are exclusive");
        return CUALIGN_EINVAL;
    }
    const int world = p->world <= 0 ? 1 : p->world;
    if (world == 1 && (p->rank != 0 || p->nccl_unique_id != nullptr)) {
        set_error("world = 1 needs rank = 0 and no NCCL id (rank=%d)", p->rank);
        return CUALIGN_EINVAL;
    }
    if (world > 1) {
        if (p->nccl_unique_id && (p->rank < 0 || p->rank >= world)) {
            set_error("NCCL shard: rank %d outside [0, %d)", p->rank, world);
            return CUALIGN_EINVAL;
        }
        if (!p->nccl_unique_id && p->rank != -1) {
            set_error("virtual shards (no NCCL id) need rank = -1 (got %d)", p->rank);
            return CUALIGN_EINVAL;
        }
        if (p->flags & CUALIGN_FLAG_EXACT) {
            set_error("CUALIGN_FLAG_EXACT is single-GPU only");
            return CUALIGN_EINVAL;
        }
    }
    return CUALIGN_OK;
}

static cualign_status open_handle(const cualign_params *params, cualign_bp **out)
{
    cualign_bp *h = new cualign_bp();
    h->alpha = params->alpha;
    h->beta = params->beta;
    h->gamma = params->gamma;
    h->flags = params->flags;
    h->dev = params->device;
    h->timing = (params->flags & CUALIGN_FLAG_TIMING) != 0;
    h->world = params->world <= 0 ? 1 : params->world;
    h->rank = params->rank < 0 ? 0 : params->rank;
    h->sched_param = params->schedule;
    h->tile_log_param = params->square_tile_log;
    *out = h;
    CA_CUDA(cudaSetDevice(h->dev));
    CA_CUDA(cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, h->dev));
    if (params->stream) {
        h->stream = (cudaStream_t)params->stream;
    } else {
        CA_CUDA(cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking));
        h->own_stream = true;
    }
    CA_CUDA(cudaStreamCreateWithFlags(&h->gstream, cudaStreamNonBlocking));
    {
        // the rounding branch gets the higher priority: its latency-bound
        // kernels are scheduled first when square-pass CTAs retire
        int lo = 0, hi = 0;
        CA_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        // CUALIGN_ROUND_PRIO (probe build): 0 = hi (default), 1 = same as
        // the iteration, 2 = lowest
        static const int rp = probe_knob("CUALIGN_ROUND_PRIO", 0);
        CA_CUDA(cudaStreamCreateWithPriority(&h->gstream2, cudaStreamNonBlocking, rp == 1 ? 0 : rp == 2 ? lo : hi));
        CA_CUDA(cudaStreamCreateWithPriority(&h->gstream3, cudaStreamNonBlocking, rp == 1 ? 0 : rp == 2 ? lo : hi));
        CA_CUDA(cudaEventCreateWithFlags(&h->eval_ev, cudaEventDisableTiming));
        CA_CUDA(cudaEventCreateWithFlags(&h->join3_ev, cudaEventDisableTiming));
    }
    for (int i = 0; i < 2; i++) {
        CA_CUDA(cudaEventCreateWithFlags(&h->sync_ev[i], cudaEventDisableTiming));
        CA_CUDA(cudaEventCreateWithFlags(&h->fork_ev[i], cudaEventDisableTiming));
    }
    return CUALIGN_OK;
}

static void close_handle(cualign_bp *h)
{
    if (!h) return;
    cudaSetDevice(h->dev);
    for (cualign_bp *s : h->vshards) close_handle(s);
    h->vshards.clear();
    nccl_free_comm(h);
    if (h->stream) cudaStreamSynchronize(h->stream);
    if (h->gstream) cudaStreamSynchronize(h->gstream);
    resolve_events(h);
    invalidate_graphs(h);
    for (auto e : h->event_pool) cudaEventDestroy(e);
    for (auto e : h->sync_ev)
        if (e) cudaEventDestroy(e);
    for (auto e : h->fork_ev)
        if (e) cudaEventDestroy(e);
    dfree_all(h);
    if (h->dist_cnt_host) cudaFreeHost(h->dist_cnt_host);
    if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
    if (h->gstream) cudaStreamDestroy(h->gstream);
    if (h->gstream2) cudaStreamDestroy(h->gstream2);
    if (h->gstream3) cudaStreamDestroy(h->gstream3);
    if (h->eval_ev) cudaEventDestroy(h->eval_ev);
    if (h->join3_ev) cudaEventDestroy(h->join3_ev);
    (void)cudaGetLastError();
    delete h;
}

static cualign_status alloc_state(cualign_bp *h)
{
    const size_t m = (size_t)h->L.m;
    for (double **p : {&h->yc, &h->zc, &h->yp, &h->zp, &h->d, &h->u}) {
        CA_TRY(dalloc(h, p, m));
        CA_CUDA(cudaMemsetAsync(*p, 0, sizeof(double) * (m ? m : 1), h->stream));
    }
    init_trace(h, "state vectors");
    if (h->world == 1 && !(h->flags & (CUALIGN_FLAG_ROUND_DAMPED | CUALIGN_FLAG_MATCH_ROUNDS)))
        CA_TRY(alloc_pipeline(h));
    init_trace(h, "pipeline buffers");
    CA_TRY(bp_setup(h));
    init_trace(h, "bp_setup");
    CA_TRY(dalloc(h, &h->p_dev, 1));
    CA_CUDA(cudaMemsetAsync(h->p_dev, 0, sizeof(int), h->stream));
    CA_TRY(ensure_gh(h, 1));
    init_trace(h, "gamma table");
    if (h->flags & CUALIGN_FLAG_EXACT) {
        CA_TRY(dalloc(h, &h->texact, m));
        CA_TRY(dalloc(h, &h->Ffull, (size_t)h->s));
        CA_TRY(ensure_sq_pos(h));
    } else {
        CA_TRY(dalloc(h, &h->tacc, m));
    }
    return CUALIGN_OK;
}

// the handle that holds the replicated rounding state (shard 0 of a group)
static cualign_bp *primary(cualign_bp *h) { return h->vshards.empty() ? h : h->vshards[0]; }

// device array [2][n_A] of the last rounding's M_y, M_z (its RoundDev slot)
static cualign_status round_mates(cualign_bp *h, const int32_t **out)
{
    int slot = 0;
    CA_CUDA(cudaMemcpyAsync(&slot, &h->rd->last_slot, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    *out = h->mates + (int64_t)slot * 2 * h->L.nA;
    return CUALIGN_OK;
}

#define API_ENTER() clear_error()
#define CHECK_H()                                   \
    do {                                            \
        if (!h) {                                   \
            set_error("handle is NULL");            \
            return CUALIGN_EINVAL;                  \
        }                                           \
        CA_CUDA(cudaSetDevice(h->dev));             \
    } while (0)

static cualign_status run_steps(cualign_bp *h, int32_t n_steps, int32_t what, RoundDev *trace);
static int default_schedule(cualign_bp *h);

// Capture (and upload) the step graphs run() will replay for the handle's
// schedule at init, so the first steps of an alignment do not pay graph
// capture / instantiation / upload.
static cualign_status precapture_step_graphs(cualign_bp *h)
{
    if (h->flags & (CUALIGN_FLAG_ROUND_DAMPED | CUALIGN_FLAG_MATCH_ROUNDS)) return CUALIGN_OK;
    const int mode = h->sched_param == 3 ? 0 : (h->sched_param > 0 ? h->sched_param : default_schedule(h));
    CA_TRY(ensure_gh(h, (int64_t)h->p + 2));
    std::vector<int> slots;
    if (mode == 2) slots = {SERIAL_SLOT};
    else if (mode == 1) {
        slots = {pslot(0, 0), pslot(0, 1), pslot(1, 0), pslot(1, 1), pslot(2, 0)};
        if (h->defer_eval) slots.insert(slots.end(), {pslot(3, 0), pslot(3, 1), pslot(4, 1)});
    }
    else slots = {CUALIGN_RUN_ITERATE | CUALIGN_RUN_ROUND};
    for (int sl : slots) {
        if (!h->graph[0][sl]) CA_TRY(capture_step(h, 0, sl));
        CA_CUDA(cudaGraphUpload(h->graph[0][sl], h->gstream));
    }
    return CUALIGN_OK;
}

} // namespace cualign

using namespace cualign;

extern "C" {

const char *cualign_last_error(void) { return g_err; }

const char *cualign_version(void) { return "cualign_bp 0.1 (sm_100a)"; }

cualign_status cualign_bp_init(const cualign_graph *A, const cualign_graph *B, const cualign_edges *L,
                               const cualign_params *params, cualign_bp **out)
{
    API_ENTER();
    if (!out) {
        set_error("out is NULL");
        return CUALIGN_EINVAL;
    }
    *out = nullptr;
    CA_TRY(check_params(params));
    if (!A || !B || !L || !A->rowptr || !B->rowptr || A->n < 0 || B->n < 0 || L->m < 0 ||
        (L->m > 0 && (!L->a || !L->b || !L->w)) || (A->n > 0 && !A->col && A->rowptr == nullptr)) {
        set_error("NULL or negative-size input");
        return CUALIGN_EINVAL;
    }
    cualign_bp *h = nullptr;
    cualign_status st = open_handle(params, &h);
    const bool virt = h && h->world > 1 && params->nccl_unique_id == nullptr;
    if (virt) {
        // in-process virtual shards (loopback exchanges) on the handle's device
        // and stream: the sharded path, testable on one GPU
        for (int r = 0; st == CUALIGN_OK && r < h->world; r++) {
            cualign_params sp = *params;
            sp.rank = r;
            sp.stream = h->stream;
            sp.nccl_unique_id = nullptr;
            cualign_bp *s = nullptr;
            st = open_handle(&sp, &s);
            if (s) h->vshards.push_back(s);
            if (st == CUALIGN_OK) st = build_problem(s, A, B, L);
            if (st == CUALIGN_OK) st = alloc_state(s);
            if (st == CUALIGN_OK) st = match_setup(s);
        }
        if (st == CUALIGN_OK) {
            // one exchange stream for the group: the loopback's copies read
            // one shard's packed halo and write another's
            for (cualign_bp *s : h->vshards) s->cstream = h->gstream2;
            cualign_bp *s0 = h->vshards[0];
            h->L = s0->L; // sizes only (the group owns no arrays itself)
            h->s_total = s0->s_total;
            h->nsq_total = s0->nsq_total;
            h->max_row = s0->max_row;
            h->fp_bits = s0->fp_bits;
            h->bounds = s0->bounds;
            st = shard_setup(h);
            if (st == CUALIGN_OK) st = shard_fsum(h); // F(S^p = 0) row sums for iteration 1
        }
    } else {
        if (st == CUALIGN_OK && h->world > 1) st = nccl_init_comm(h, params->nccl_unique_id);
        if (h && h->world > 1) h->cstream = h->gstream2; // the shard's exchange stream
        init_trace(h, "^start");
        if (st == CUALIGN_OK) st = build_problem(h, A, B, L);
        init_trace(h, "build_problem");
        if (st == CUALIGN_OK) st = alloc_state(h);
        init_trace(h, "alloc_state");
        if (st == CUALIGN_OK) st = match_setup(h);
        init_trace(h, "match_setup");
        if (st == CUALIGN_OK && h->world > 1) st = shard_setup(h);
        if (st == CUALIGN_OK) st = h->world > 1 ? shard_fsum(h) : bp_fsum(h); // F(S^p = 0) sums for iteration 1
        if (st == CUALIGN_OK && h->world == 1) st = bp_top2(h);                 // othermax inputs of iteration 1
        init_trace(h, "fsum");
        // pipelined graphs evaluate each round one step later (probe build:
        // CUALIGN_PIPE_DEFER_EVAL=0 keeps evaluate in the round's own graph)
        if (st == CUALIGN_OK) h->defer_eval = can_defer_eval(h) && probe_knob("CUALIGN_PIPE_DEFER_EVAL", 1) != 0;
        if (st == CUALIGN_OK && h->world == 1) st = precapture_step_graphs(h);
        init_trace(h, "step graphs");
    }
    if (st == CUALIGN_OK) {
        cudaError_t e = cudaStreamSynchronize(h->stream);
        if (e != cudaSuccess) {
            set_error("init: %s", cudaGetErrorString(e));
            st = CUALIGN_ECUDA;
        }
    }
    if (st != CUALIGN_OK) {
        std::string msg = g_err;
        close_handle(h);
        set_error("%s", msg.c_str());
        return st;
    }
    *out = h;
    return CUALIGN_OK;
}

cualign_status cualign_bp_iterate(cualign_bp *h, int32_t n_steps)
{
    API_ENTER();
    CHECK_H();
    if (n_steps < 0) {
        set_error("n_steps < 0");
        return CUALIGN_EINVAL;
    }
    return h->world > 1 ? shard_iterate(h, n_steps) : bp_iterate(h, n_steps);
}

cualign_status cualign_bp_run(cualign_bp *h, int32_t n_steps, int32_t what)
{
    API_ENTER();
    CHECK_H();
    if (n_steps < 0) {
        set_error("n_steps < 0");
        return CUALIGN_EINVAL;
    }
    if (n_steps == 0) return CUALIGN_OK;
    if (what < 1 || what > 3) {
        set_error("run: what must be CUALIGN_RUN_ITERATE, CUALIGN_RUN_ROUND or both");
        return CUALIGN_EINVAL;
    }
    return run_steps(h, n_steps, what, nullptr);
}

// thread-local pinned staging for run_trace (cached: pinned allocation is slow)
struct PinnedTrace {
    RoundDev *p = nullptr;
    size_t n = 0;
    ~PinnedTrace()
    {
        if (p) cudaFreeHost(p);
    }
};

cualign_status cualign_bp_run_trace(cualign_bp *h, int32_t n_steps, cualign_round_info *infos)
{
    API_ENTER();
    CHECK_H();
    if (n_steps < 0 || (n_steps > 0 && !infos)) {
        set_error("run_trace: n_steps < 0 or infos is NULL");
        return CUALIGN_EINVAL;
    }
    if (n_steps == 0) return CUALIGN_OK;
    static thread_local PinnedTrace pt;
    if (pt.n < (size_t)n_steps) {
        if (pt.p) cudaFreeHost(pt.p);
        pt.p = nullptr;
        pt.n = 0;
        CA_CUDA(cudaHostAlloc((void **)&pt.p, sizeof(RoundDev) * (size_t)n_steps, cudaHostAllocDefault));
        pt.n = (size_t)n_steps;
    }
    CA_TRY(run_steps(h, n_steps, CUALIGN_RUN_ITERATE | CUALIGN_RUN_ROUND, pt.p));
    cualign_bp *q = primary(h);
    CA_CUDA(cudaStreamSynchronize(q->stream));
    CA_CUDA(cudaStreamSynchronize(q->gstream));
    for (int32_t k = 0; k < n_steps; k++) {
        infos[k] = pt.p[k].info;
        infos[k].best_score = pt.p[k].best_score;
        infos[k].best_iter = pt.p[k].best_iter;
    }
    q->last_info = infos[n_steps - 1];
    return CUALIGN_OK;
}

} // extern "C"

namespace cualign {
// Step schedule of run() when the caller leaves it to the library (no timed
// selection on the critical path).  Measured with the round-2 kernels
// (tools/probe_schedules.py, profiles/r02_schedules.jsonl; ms per step after
// 40 warm steps, pipelined / serial): T 0.041 / 0.047, P 0.121 / 0.133 --
// launch- and latency-bound steps gain from overlapping the rounding with the
// next iteration; O 0.672 / 0.678 (bench: 1544 / 1487 it/s over 300 steps,
// 1435 / 1396 in the 20-step window) -- a long square pass (s/m = 20) hides
// the rounding; R k = 5 0.856 / 0.773 (s/m = 5: the step is short next to
// its rounding, which then contends with it), S 5.57 / 5.47 and R k = 50
// 6.37 / 6.08 (s >= 8.4e8: the HBM-bound pass is delayed by any traffic
// beside it).  Pipelined below 10^7 nonzeros of S, and up to 3e8 nonzeros
// when s/m >= 10; serial otherwise.
// With the deferred evaluate (the pipelined graphs evaluate each round one
// step later, can_defer_eval) pipelined wins or ties on every config
// (profiles/r02_schedules_deferred.jsonl, pipelined / serial ms per step):
// T 0.036 / 0.052, P 0.107 / 0.132, O 0.633 / 0.677, R k = 5 0.696 / 0.768,
// S 5.49 / 5.54, R k = 50 6.149 / 6.139; the size rule (measured before it,
// comment above) stays for handles
// whose rounding cannot be deferred (damped rounding, pointer rounds, B-side
// proposers).
static int default_schedule(cualign_bp *h)
{
    if (can_defer_eval(h)) return 1;
    const int64_t s = h->s_total ? h->s_total : h->s;
    const int64_t m = h->L.m > 0 ? h->L.m : 1;
    if (s < 10000000) return 1;
    return (s < 300000000 && s >= 10 * m) ? 1 : 2;
}

// The sharded iteration (k_edge, top-2 all-gather, u halo on the exchange
// stream beside the owned-f squares, remote-f squares, F halo; NCCL calls
// are capturable) as ONE graph, replayed by run(): no host work per kernel or
// exchange.  Captured on the group's capture stream with every shard's main
// stream pointed at it; re-captured when a shard's gamma table moves.
static cualign_status shard_iterate_graph(cualign_bp *h)
{
    // NCCL connects peers lazily, at a channel's first use -- which must not
    // happen inside a stream capture: the first sharded step of a handle runs
    // eagerly, the graph is captured at the second
    if (!h->shard_warm) {
        h->shard_warm = true;
        return shard_iterate(h, 1);
    }
    std::vector<cualign_bp *> S = h->vshards.empty() ? std::vector<cualign_bp *>{h} : h->vshards;
    for (cualign_bp *s : S) CA_TRY(ensure_gh(s, (int64_t)s->p + 2));
    std::vector<const void *> gh;
    for (cualign_bp *s : S) gh.push_back(s->gh_dev);
    if (h->shard_graph && gh != h->shard_graph_gh) {
        cudaGraphExecDestroy(h->shard_graph);
        h->shard_graph = nullptr;
    }
    if (!h->shard_graph) {
        struct Saved {
            cudaStream_t stream;
            int32_t p;
            int64_t launches, class_launches[CUALIGN_NUM_KERNEL_CLASSES], comm_calls, comm_bytes_in;
        };
        std::vector<Saved> saved;
        for (cualign_bp *s : S) {
            Saved v{s->stream, s->p, s->launches, {}, s->comm_calls, s->comm_bytes_in};
            for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) v.class_launches[c] = s->class_launches[c];
            saved.push_back(v);
            s->stream = h->gstream;
            s->capturing = true;
        }
        const int32_t hp = h->p;
        cualign_status st = CUALIGN_OK;
        cudaGraph_t g = nullptr;
        if (cudaStreamBeginCapture(h->gstream, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
            set_error("sharded step: graph capture could not start");
            st = CUALIGN_ECUDA;
        } else {
            st = shard_iterate(h, 1);
            const cudaError_t e2 = cudaStreamEndCapture(h->gstream, &g);
            if (st == CUALIGN_OK && e2 != cudaSuccess) {
                set_error("sharded step capture: %s", cudaGetErrorString(e2));
                st = CUALIGN_ECUDA;
            }
            if (st == CUALIGN_OK && cudaGraphInstantiate(&h->shard_graph, g, 0) != cudaSuccess) {
                set_error("sharded step: graph instantiate failed");
                st = CUALIGN_ECUDA;
            }
            if (g) cudaGraphDestroy(g);
        }
        // what one replay launches / exchanges (per shard), then the counters
        // as they were: the capture ran nothing
        h->shard_step_counts.assign(S.size(), {});
        for (size_t i = 0; i < S.size(); i++) {
            cualign_bp *s = S[i];
            auto &c = h->shard_step_counts[i];
            c.launches = s->launches - saved[i].launches;
            for (int k = 0; k < CUALIGN_NUM_KERNEL_CLASSES; k++)
                c.class_launches[k] = s->class_launches[k] - saved[i].class_launches[k];
            c.comm_calls = s->comm_calls - saved[i].comm_calls;
            c.comm_bytes_in = s->comm_bytes_in - saved[i].comm_bytes_in;
            s->stream = saved[i].stream;
            s->p = saved[i].p;
            s->launches = saved[i].launches;
            for (int k = 0; k < CUALIGN_NUM_KERNEL_CLASSES; k++) s->class_launches[k] = saved[i].class_launches[k];
            s->comm_calls = saved[i].comm_calls;
            s->comm_bytes_in = saved[i].comm_bytes_in;
            s->capturing = false;
        }
        h->p = hp;
        (void)cudaGetLastError();
        CA_TRY(st);
        h->shard_graph_gh = gh;
    }
    CA_CUDA(cudaEventRecord(h->sync_ev[0], h->stream));
    CA_CUDA(cudaStreamWaitEvent(h->gstream, h->sync_ev[0], 0));
    CA_CUDA(cudaGraphLaunch(h->shard_graph, h->gstream));
    CA_CUDA(cudaEventRecord(h->sync_ev[1], h->gstream));
    CA_CUDA(cudaStreamWaitEvent(h->stream, h->sync_ev[1], 0));
    for (size_t i = 0; i < S.size(); i++) {
        cualign_bp *s = S[i];
        const auto &c = h->shard_step_counts[i];
        s->p += 1;
        s->launches += c.launches;
        for (int k = 0; k < CUALIGN_NUM_KERNEL_CLASSES; k++) s->class_launches[k] += c.class_launches[k];
        s->comm_calls += c.comm_calls;
        s->comm_bytes_in += c.comm_bytes_in;
    }
    if (!h->vshards.empty()) h->p += 1;
    return CUALIGN_OK;
}

static cualign_status run_steps(cualign_bp *h, int32_t n_steps, int32_t what, RoundDev *trace)
{
    if (h->world > 1) {
        // sharded: the iteration replayed from its graph (eager with timing
        // on: per-exchange events), the rounding's merge batches on the host
        cualign_bp *q = primary(h);
        for (int32_t k = 0; k < n_steps; k++) {
            // graph replay for in-process shards; process shards (NCCL) step
            // eagerly: NCCL calls are capturable, but with the only transport
            // this sandbox can test (ranks sharing one GPU over sockets) a
            // captured step deadlocked, so it stays unvalidated and off
            const bool graph = !h->timing && !h->vshards.empty();
            if (what & CUALIGN_RUN_ITERATE) CA_TRY(graph ? shard_iterate_graph(h) : shard_iterate(h, 1));
            if (what & CUALIGN_RUN_ROUND) CA_TRY(shard_round(h));
            if (trace)
                CA_CUDA(cudaMemcpyAsync(trace + k, q->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, q->stream));
        }
        h->have_info = h->have_info || (what & CUALIGN_RUN_ROUND);
        return CUALIGN_OK;
    }
    // both halves of a step: schedules 0 = one graph per step with the
    // rounding forked beside the square pass, 1 = pipelined (rounding of k
    // beside iteration k+1), 2 = serial (one graph: iteration, then its
    // rounding); results are identical whichever runs (tests compare them
    // with the eager sequence bit for bit).  Not pipelined when the rounding
    // reads y^p, z^p (ROUND_DAMPED: the next iteration overwrites them) or
    // the matching is the cooperative pointer-round kernel (MATCH_ROUNDS: its
    // grid must be co-resident).  The caller picks one with
    // cualign_params.schedule, else default_schedule().
    // cualign_params.schedule: 1 pipelined, 2 serial, 3 forked (pipe_mode 0)
    const int pipe_env = h->sched_param == 3 ? 0 : (h->sched_param > 0 ? h->sched_param : -1);
    const bool both = what == (CUALIGN_RUN_ITERATE | CUALIGN_RUN_ROUND) &&
                      !(h->flags & (CUALIGN_FLAG_ROUND_DAMPED | CUALIGN_FLAG_MATCH_ROUNDS));
    auto run_plain = [&](int32_t n, RoundDev *tr) -> cualign_status {
        if (!tr) return run_graph(h, n, what);
        for (int32_t k = 0; k < n; k++) {
            CA_TRY(run_graph(h, 1, what));
            CA_CUDA(cudaMemcpyAsync(tr + k, h->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, h->stream));
        }
        return CUALIGN_OK;
    };
    auto run_serial = [&](int32_t n, RoundDev *tr) -> cualign_status {
        if (n <= 0) return CUALIGN_OK;
        CA_TRY(ensure_gh(h, (int64_t)h->p + n + 1));
        CA_CUDA(cudaEventRecord(h->sync_ev[0], h->stream));
        CA_CUDA(cudaStreamWaitEvent(h->gstream, h->sync_ev[0], 0));
        for (int32_t k = 0; k < n; k++) {
            CA_TRY(launch_slot(h, SERIAL_SLOT));
            h->p += 1;
            if (tr) CA_CUDA(cudaMemcpyAsync(tr + k, h->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, h->gstream));
        }
        h->have_info = true;
        CA_CUDA(cudaEventRecord(h->sync_ev[1], h->gstream));
        CA_CUDA(cudaStreamWaitEvent(h->stream, h->sync_ev[1], 0));
        return CUALIGN_OK;
    };
    auto run_mode = [&](int mode, int32_t n, RoundDev *tr) -> cualign_status {
        if (mode == 1) return run_pipelined(h, n, tr);
        if (mode == 2) return run_serial(n, tr);
        return run_plain(n, tr);
    };
    if (!both) return run_plain(n_steps, trace);
    if (pipe_env >= 0 && pipe_env <= 2) {
        h->pipe_mode = pipe_env; // given by the caller (reported as chosen)
        return run_mode(pipe_env, n_steps, trace);
    }
    if (h->pipe_mode < 0) h->pipe_mode = default_schedule(h);
    return run_mode(h->pipe_mode, n_steps, trace);
}
} // namespace cualign

extern "C" {

cualign_status cualign_bp_set_timing(cualign_bp *h, int32_t on)
{
    API_ENTER();
    CHECK_H();
    h->timing = on != 0;
    for (cualign_bp *s : h->vshards) s->timing = on != 0;
    return CUALIGN_OK;
}

cualign_status cualign_bp_round(cualign_bp *h, cualign_round_info *info)
{
    API_ENTER();
    CHECK_H();
    CA_TRY(h->world > 1 ? shard_round(h) : match_round(h));
    h->have_info = true;
    if (info) {
        cualign_bp *q = primary(h);
        CA_CUDA(cudaMemcpyAsync(&q->last_info, &q->rd->info, sizeof(cualign_round_info), cudaMemcpyDeviceToHost,
                                q->stream));
        CA_CUDA(cudaStreamSynchronize(q->stream));
        *info = q->last_info;
    }
    return CUALIGN_OK;
}

cualign_status cualign_bp_get_best(cualign_bp *h, int32_t *mate_a, cualign_round_info *info)
{
    API_ENTER();
    CHECK_H();
    h = primary(h); // rounding is replicated on every shard
    RoundDev r;
    CA_CUDA(cudaMemcpyAsync(&r, h->rd, sizeof(RoundDev), cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    if (mate_a && h->L.nA) {
        // bestM lives in its round's mate slot (RoundDev); empty until a score > 0
        if (r.best_iter > 0)
            CA_CUDA(cudaMemcpy(mate_a, h->mates + ((int64_t)r.best_slot * 2 + r.best_source) * h->L.nA,
                               sizeof(int32_t) * (size_t)h->L.nA, cudaMemcpyDeviceToHost));
        else
            for (int32_t a = 0; a < h->L.nA; a++) mate_a[a] = -1;
    }
    if (info) {
        *info = r.info;
        info->best_score = r.best_score;
        info->best_iter = r.best_iter;
    }
    return CUALIGN_OK;
}

void cualign_bp_free(cualign_bp *h) { close_handle(h); }

cualign_status cualign_bp_get_sizes(cualign_bp *h, cualign_sizes *sz)
{
    API_ENTER();
    CHECK_H();
    if (!sz) {
        set_error("sizes is NULL");
        return CUALIGN_EINVAL;
    }
    CA_CUDA(cudaStreamSynchronize(h->stream));
    cualign_bp *q = primary(h);
    sz->n_a = q->L.nA;
    sz->n_b = q->L.nB;
    sz->m = q->L.m;
    sz->s = q->s_total;
    sz->squares = q->nsq_total;
    sz->max_row = q->max_row;
    sz->p = h->p;
    sz->fixed_point_bits = (q->flags & CUALIGN_FLAG_EXACT) ? 0 : q->fp_bits;
    sz->device_bytes = h->device_bytes;
    for (cualign_bp *s : h->vshards) sz->device_bytes += s->device_bytes;
    sz->rank = h->vshards.empty() ? h->rank : -1;
    sz->world = h->world;
    sz->edge_begin = h->vshards.empty() ? h->e0 : 0;
    sz->edge_end = h->vshards.empty() ? h->e1 : q->L.m;
    sz->squares_local = h->vshards.empty() ? h->nsq : q->nsq_total;
    sz->merge_rounds = q->dist_rounds;
    sz->schedule = h->pipe_mode;
    return CUALIGN_OK;
}

cualign_status cualign_bp_get_S(cualign_bp *h, int64_t *rowptr, int32_t *col, int64_t *s_out)
{
    API_ENTER();
    CHECK_H();
    if (!h->vshards.empty()) {
        // virtual shards own consecutive rows: concatenate their CSRs
        int64_t off = 0;
        for (cualign_bp *s : h->vshards) {
            const int64_t ml = s->e1 - s->e0;
            if (rowptr) {
                std::vector<int64_t> rp((size_t)ml + 1);
                CA_CUDA(cudaMemcpy(rp.data(), s->Srp, sizeof(int64_t) * (size_t)(ml + 1), cudaMemcpyDeviceToHost));
                for (int64_t i = 0; i <= ml; i++) rowptr[s->e0 + i] = rp[(size_t)i] + off;
            }
            if (col && s->s)
                CA_CUDA(cudaMemcpy(col + off, s->Scol, sizeof(int32_t) * (size_t)s->s, cudaMemcpyDeviceToHost));
            off += s->s;
        }
        if (s_out) *s_out = off;
        return CUALIGN_OK;
    }
    if (h->world > 1) {
        set_error("get_S: a process shard holds only its own rows; use virtual shards or world = 1");
        return CUALIGN_ESTATE;
    }
    CA_TRY(ensure_csr(h));
    if (rowptr)
        CA_CUDA(cudaMemcpyAsync(rowptr, h->Srp, sizeof(int64_t) * ((size_t)h->L.m + 1), cudaMemcpyDeviceToHost,
                                h->stream));
    if (col && h->s)
        CA_CUDA(cudaMemcpyAsync(col, h->Scol, sizeof(int32_t) * (size_t)h->s, cudaMemcpyDeviceToHost, h->stream));
    CA_CUDA(cudaStreamSynchronize(h->stream));
    if (s_out) *s_out = h->s;
    return CUALIGN_OK;
}

cualign_status cualign_bp_get_state(cualign_bp *h, double *yc, double *zc, double *yp, double *zp, double *d,
                                    double *Sp, int32_t *p)
{
    API_ENTER();
    CHECK_H();
    if (h->world > 1) {
        if (Sp) {
            set_error("get_state: S^p of a sharded handle is distributed (pass Sp = NULL)");
            return CUALIGN_ESTATE;
        }
        // every per-edge vector is valid on its owner's slice: assemble the
        // slices (virtual shards) or return this process shard's arrays (its
        // owned slice [edge_begin, edge_end) valid)
        std::vector<cualign_bp *> S = h->vshards.empty() ? std::vector<cualign_bp *>{h} : h->vshards;
        CA_CUDA(cudaStreamSynchronize(S[0]->stream));
        for (cualign_bp *s : S) {
            const int64_t a = h->vshards.empty() ? 0 : s->e0, b = h->vshards.empty() ? s->L.m : s->e1;
            const size_t nb = sizeof(double) * (size_t)(b - a);
            if (!nb) continue;
            if (yc) CA_CUDA(cudaMemcpy(yc + a, s->yc + a, nb, cudaMemcpyDeviceToHost));
            if (zc) CA_CUDA(cudaMemcpy(zc + a, s->zc + a, nb, cudaMemcpyDeviceToHost));
            if (yp) CA_CUDA(cudaMemcpy(yp + a, s->yp + a, nb, cudaMemcpyDeviceToHost));
            if (zp) CA_CUDA(cudaMemcpy(zp + a, s->zp + a, nb, cudaMemcpyDeviceToHost));
            if (d) CA_CUDA(cudaMemcpy(d + a, s->d + a, nb, cudaMemcpyDeviceToHost));
        }
        if (p) *p = h->p;
        return CUALIGN_OK;
    }
    const size_t mb = sizeof(double) * (size_t)h->L.m;
    struct {
        double *dst;
        double *src;
    } vec[] = {{yc, h->yc}, {zc, h->zc}, {yp, h->yp}, {zp, h->zp}, {d, h->d}};
    for (auto &v : vec)
        if (v.dst && mb) CA_CUDA(cudaMemcpyAsync(v.dst, v.src, mb, cudaMemcpyDeviceToHost, h->stream));
    if (Sp && h->s) {
        TmpBuf tb;
        CA_CUDA(tmalloc(h, tb, sizeof(double) * (size_t)h->s));
        double *tmp = (double *)tb.p;
        cualign_status st = bp_scatter_Sp(h, tmp);
        if (st == CUALIGN_OK) {
            cudaError_t e = cudaMemcpyAsync(Sp, tmp, sizeof(double) * (size_t)h->s, cudaMemcpyDeviceToHost, h->stream);
            if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
            if (e != cudaSuccess) {
                set_error("get_state: %s", cudaGetErrorString(e));
                st = CUALIGN_ECUDA;
            }
        }
        CA_TRY(st);
    }
    CA_CUDA(cudaStreamSynchronize(h->stream));
    if (p) *p = h->p;
    return CUALIGN_OK;
}

cualign_status cualign_bp_set_state(cualign_bp *h, const double *yp, const double *zp, const double *Sp,
                                    int32_t p)
{
    API_ENTER();
    CHECK_H();
    if (h->world > 1) {
        set_error("set_state is single-GPU only");
        return CUALIGN_ESTATE;
    }
    if (!yp || !zp || (!Sp && h->s) || p < 0) {
        set_error("set_state: NULL buffer or p < 0");
        return CUALIGN_EINVAL;
    }
    const size_t mb = sizeof(double) * (size_t)h->L.m;
    if (mb) {
        CA_CUDA(cudaMemcpyAsync(h->yp, yp, mb, cudaMemcpyHostToDevice, h->stream));
        CA_CUDA(cudaMemcpyAsync(h->zp, zp, mb, cudaMemcpyHostToDevice, h->stream));
    }
    if (h->s) {
        TmpBuf tb;
        CA_CUDA(tmalloc(h, tb, sizeof(double) * (size_t)h->s));
        double *tmp = (double *)tb.p;
        cudaError_t e = cudaMemcpyAsync(tmp, Sp, sizeof(double) * (size_t)h->s, cudaMemcpyHostToDevice, h->stream);
        cualign_status st = CUALIGN_OK;
        if (e != cudaSuccess) {
            set_error("set_state: %s", cudaGetErrorString(e));
            st = CUALIGN_ECUDA;
        }
        if (st == CUALIGN_OK) st = bp_gather_Sp(h, tmp);
        if (st == CUALIGN_OK && cudaStreamSynchronize(h->stream) != cudaSuccess) st = CUALIGN_ECUDA;
        CA_TRY(st);
    }
    h->p = p;
    CA_TRY(ensure_gh(h, (int64_t)p + 1));
    CA_CUDA(cudaMemcpyAsync(h->p_dev, &h->p, sizeof(int), cudaMemcpyHostToDevice, h->stream));
    CA_TRY(bp_fsum(h));
    CA_TRY(bp_top2(h)); // othermax inputs of the next iteration from the injected y^p, z^p
    CA_CUDA(cudaStreamSynchronize(h->stream));
    return CUALIGN_OK;
}

cualign_status cualign_bp_get_round_mates(cualign_bp *h, int32_t *mate_y, int32_t *mate_z)
{
    API_ENTER();
    CHECK_H();
    cualign_bp *q = primary(h);
    if (!h->have_info && !q->have_info) {
        set_error("get_round_mates: no rounding has run on this handle");
        return CUALIGN_ESTATE;
    }
    CA_CUDA(cudaStreamSynchronize(h->stream));
    CA_CUDA(cudaStreamSynchronize(q->stream));
    const size_t nb = sizeof(int32_t) * (size_t)q->L.nA;
    const int32_t *src = nullptr;
    CA_TRY(round_mates(q, &src));
    if (nb && mate_y) CA_CUDA(cudaMemcpy(mate_y, src, nb, cudaMemcpyDeviceToHost));
    if (nb && mate_z) CA_CUDA(cudaMemcpy(mate_z, src + q->L.nA, nb, cudaMemcpyDeviceToHost));
    return CUALIGN_OK;
}

cualign_status cualign_bp_sample_squares(cualign_bp *h, const int32_t *edges, int64_t n, int64_t cap,
                                         int32_t *e_out, int32_t *f_out, double *v_ef, double *v_fe,
                                         int64_t *n_out)
{
    API_ENTER();
    CHECK_H();
    if (!n_out || n < 0 || (n > 0 && !edges)) {
        set_error("sample_squares: NULL n_out / edges or n < 0");
        return CUALIGN_EINVAL;
    }
    if (h->world > 1 && h->vshards.empty()) {
        set_error("sample_squares: a process shard holds only its own squares");
        return CUALIGN_ESTATE;
    }
    CA_CUDA(cudaStreamSynchronize(h->stream));
    std::vector<cualign_bp *> S = h->vshards.empty() ? std::vector<cualign_bp *>{h} : h->vshards;
    int64_t total = 0;
    for (cualign_bp *s : S) {
        int64_t k = 0;
        const int64_t off = total < cap ? total : cap;
        CA_TRY(bp_sample_squares(s, edges, n, cap - off, e_out ? e_out + off : nullptr, f_out ? f_out + off : nullptr,
                                 v_ef ? v_ef + off : nullptr, v_fe ? v_fe + off : nullptr, &k));
        total += k;
    }
    *n_out = total;
    return CUALIGN_OK;
}

cualign_status cualign_bp_get_stats(cualign_bp *h, cualign_stats *stats, int32_t reset)
{
    API_ENTER();
    CHECK_H();
    CA_CUDA(cudaStreamSynchronize(h->stream));
    std::vector<cualign_bp *> S{h};
    for (cualign_bp *s : h->vshards) S.push_back(s);
    if (stats) {
        stats->launches = 0;
        for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) {
            stats->class_launches[c] = 0;
            stats->class_ms[c] = 0.0;
        }
    }
    if (stats) {
        stats->comm_calls = 0;
        stats->comm_bytes_in = 0;
        stats->comm_ms = 0.0;
    }
    for (cualign_bp *s : S) {
        resolve_events(s);
        for (auto &ep : s->comm_events) {
            float ms = 0.f;
            if (cudaEventSynchronize(ep.b) == cudaSuccess && cudaEventElapsedTime(&ms, ep.a, ep.b) == cudaSuccess)
                s->comm_ms += ms;
            s->event_pool.push_back(ep.a);
            s->event_pool.push_back(ep.b);
        }
        s->comm_events.clear();
        (void)cudaGetLastError();
        if (stats) {
            stats->comm_calls += s->comm_calls;
            stats->comm_bytes_in += s->comm_bytes_in;
            stats->comm_ms += s->comm_ms;
            stats->launches += s->launches;
            for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) {
                stats->class_launches[c] += s->class_launches[c];
                stats->class_ms[c] += s->class_ms[c];
            }
        }
        if (reset) {
            s->comm_calls = 0;
            s->comm_bytes_in = 0;
            s->comm_ms = 0.0;
            s->launches = 0;
            for (int c = 0; c < CUALIGN_NUM_KERNEL_CLASSES; c++) {
                s->class_launches[c] = 0;
                s->class_ms[c] = 0.0;
            }
        }
    }
    return CUALIGN_OK;
}

cualign_status cualign_nccl_unique_id(void *id, int32_t len)
{
    API_ENTER();
    if (!id) {
        set_error("id is NULL");
        return CUALIGN_EINVAL;
    }
    return nccl_unique_id(id, len);
}

cualign_status cualign_match(const cualign_edges *L, int32_t n_a, int32_t n_b, const double *x,
                             const cualign_params *params, int32_t *mate_a, int32_t *mate_b, int32_t *rounds_out)
{
    API_ENTER();
    if (!L || !x || !params || n_a < 0 || n_b < 0 || L->m < 0 || (L->m > 0 && (!L->a || !L->b))) {
        set_error("cualign_match: NULL or negative-size input");
        return CUALIGN_EINVAL;
    }
    cualign_params prm = *params;
    prm.alpha = 1.0;
    prm.beta = 0.0;
    prm.gamma = 1.0;
    prm.rank = 0;
    prm.world = 1;
    prm.nccl_unique_id = nullptr;
    cualign_bp *h = nullptr;
    cualign_status st = open_handle(&prm, &h);
    const bool devp = (prm.flags & CUALIGN_FLAG_DEVICE_PTRS) != 0;
    cualign_edges E = *L;
    E.w = nullptr;
    double *xd = nullptr;
    if (st == CUALIGN_OK) st = build_L(h, h->L, &E, devp, true, n_a, n_b);
    if (st == CUALIGN_OK) st = match_setup(h);
    if (st == CUALIGN_OK) st = dalloc(h, &xd, (size_t)L->m);
    if (st == CUALIGN_OK && L->m) {
        if (cudaMemcpyAsync(xd, x, sizeof(double) * (size_t)L->m,
                            devp ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, h->stream) != cudaSuccess) {
            set_error("cualign_match: copy of x failed");
            st = CUALIGN_ECUDA;
        }
    }
    if (st == CUALIGN_OK) st = match_standalone(h, xd, rounds_out);
    int ws = 0;
    if (st == CUALIGN_OK && (cudaMemcpyAsync(&ws, &h->rd->wslot, sizeof(int), cudaMemcpyDeviceToHost, h->stream) !=
                                 cudaSuccess ||
                             cudaStreamSynchronize(h->stream) != cudaSuccess))
        st = CUALIGN_ECUDA;
    if (st == CUALIGN_OK && mate_a && n_a)
        if (cudaMemcpyAsync(mate_a, h->mates + (int64_t)ws * 2 * n_a, sizeof(int32_t) * (size_t)n_a,
                            cudaMemcpyDeviceToHost, h->stream) != cudaSuccess)
            st = CUALIGN_ECUDA;
    if (st == CUALIGN_OK && mate_b && n_b)
        if (cudaMemcpyAsync(mate_b, h->mateB, sizeof(int32_t) * (size_t)n_b, cudaMemcpyDeviceToHost, h->stream) !=
            cudaSuccess)
            st = CUALIGN_ECUDA;
    if (st == CUALIGN_OK) {
        cudaError_t e = cudaStreamSynchronize(h->stream);
        if (e != cudaSuccess) {
            set_error("cualign_match: %s", cudaGetErrorString(e));
            st = CUALIGN_ECUDA;
        }
    }
    std::string msg = g_err;
    close_handle(h);
    if (st != CUALIGN_OK) set_error("%s", msg.c_str());
    return st;
}

cualign_status cualign_quality_eval(const cualign_graph *A, const cualign_graph *B, const int32_t *map_ab,
                                    const int32_t *truth, const cualign_params *params, cualign_quality *out)
{
    API_ENTER();
    if (!A || !B || !params || !out || (A->n > 0 && !map_ab)) {
        set_error("cualign_quality_eval: NULL input");
        return CUALIGN_EINVAL;
    }
    cualign_params prm = *params;
    prm.alpha = 1.0;
    prm.beta = 0.0;
    prm.gamma = 1.0;
    prm.rank = 0;
    prm.world = 1;
    prm.nccl_unique_id = nullptr;
    prm.flags &= (CUALIGN_FLAG_DEVICE_PTRS | CUALIGN_FLAG_TIMING);
    cualign_bp *h = nullptr;
    cualign_status st = open_handle(&prm, &h);
    if (st == CUALIGN_OK) st = quality_eval(h, A, B, map_ab, truth, out);
    std::string msg = g_err;
    close_handle(h);
    if (st != CUALIGN_OK) set_error("%s", msg.c_str());
    return st;
}

cualign_status cualign_knn(const float *YA, int32_t n_a, const float *YB, int32_t n_b, int32_t d, int32_t k,
                           const cualign_params *params, int32_t *L_a, int32_t *L_b, double *L_w)
{
    API_ENTER();
    if (!params || n_a < 0 || n_b < 0 || (n_a > 0 && (!YA || !L_a || !L_b || !L_w)) || (n_b > 0 && !YB)) {
        set_error("cualign_knn: NULL or negative-size input");
        return CUALIGN_EINVAL;
    }
    if (d < 1 || d > 256 || k < 1 || k > 32 || (n_a > 0 && k > n_b)) {
        set_error("cualign_knn: need 1 <= d <= 256, 1 <= k <= min(32, n_b) (d = %d, k = %d, n_b = %d)", d, k, n_b);
        return CUALIGN_EINVAL;
    }
    cualign_params prm = *params;
    prm.alpha = 1.0;
    prm.beta = 0.0;
    prm.gamma = 1.0;
    prm.rank = 0;
    prm.world = 1;
    prm.nccl_unique_id = nullptr;
    prm.flags &= (CUALIGN_FLAG_DEVICE_PTRS | CUALIGN_FLAG_TIMING);
    cualign_bp *h = nullptr;
    cualign_status st = open_handle(&prm, &h);
    if (st == CUALIGN_OK) st = knn_build(h, YA, n_a, YB, n_b, d, k, L_a, L_b, L_w);
    std::string msg = g_err;
    close_handle(h);
    if (st != CUALIGN_OK) set_error("%s", msg.c_str());
    return st;
}

} // extern "C"
