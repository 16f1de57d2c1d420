/*
 * cualign_bp.h -- C ABI of the B200-native NetAlignBP + matching engine.
 *
 * Method: cuAlign (Xiang, Khan, Ferdous, Aravind, Halappanavar, SC-W 2023),
 * /root/reference/PAPER.md.  The engine runs the data-parallel hot path of
 * the paper's Alg. 2 on one B200 (sm_100a):
 *
 *   init     a1  canonical L (A-side rows, B-side incidence)
 *            a2  overlap matrix S (Alg. 3) + its square layout PAPER.md:66, :181, :185-197
 *   iterate  a3  F = bound_{0,beta}[beta S + S^p'], d = alpha w + F e   (Alg. 2 l.9-10, :162-163)
 *            a4  y^c = d - othermaxcol(z^p), z^c = d - othermaxrow(y^p) (l.11-12, :164-165, :203)
 *            a5  S^c = diag(y^c + z^c - d) S - F                        (l.13, :166)
 *            a6  damping with gamma^p                                   (l.14-16, :167-169)
 *   round    a7  1/2-approx. locally-dominant matching on y^c and z^c  (l.17-20, :170-173, :207-209)
 *            a8  evaluate alpha*w(M) + beta*x'Sx/2, keep the best      (l.21-24, :174-177, Eq. 1 :64-72)
 *
 * Readings of the paper where it is silent or garbled are listed in DESIGN.md
 * (Z1-Z27); the ones that change results are selectable through flags.
 *
 * Conventions (all functions):
 *   - Every function returns a cualign_status and never throws; on error a
 *     human-readable message is available from cualign_last_error()
 *     (thread-local, valid until the next call on the same thread).
 *   - Inputs are borrowed for the duration of the call and copied; outputs are
 *     written to caller-owned buffers; the handle owns all device memory it
 *     allocates until cualign_bp_free().
 *   - Pointers are HOST pointers unless CUALIGN_FLAG_DEVICE_PTRS is set in
 *     cualign_params.flags, in which case the graph / edge arrays given to
 *     cualign_bp_init are device pointers on params.device.  State / output
 *     buffers of the get/set functions are always host pointers.
 *   - cualign_bp_iterate() is asynchronous on params.stream; CUDA errors
 *     surface at the next synchronising call.  cualign_bp_round() with a
 *     non-NULL info, every get_* function and cualign_bp_free() synchronise.
 *   - One handle per host thread; distinct handles are independent.
 *   - Sizes are int64; vertex ids and edge ids are int32 (m < 2^31), S row
 *     pointers int64 (nnz(S) may exceed 2^31).
 */
#ifndef CUALIGN_BP_H
#define CUALIGN_BP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct cualign_bp cualign_bp; /* opaque handle; owns all device state */

typedef enum {
    CUALIGN_OK = 0,
    CUALIGN_EINVAL = -1, /* invalid argument / malformed input (message says which) */
    CUALIGN_ENOMEM = -2, /* device allocation failed */
    CUALIGN_ECUDA = -3,  /* a CUDA runtime call failed */
    CUALIGN_ENCCL = -4,  /* an NCCL call failed (sharded handles) */
    CUALIGN_ESTATE = -5  /* call not valid in the handle's current state */
} cualign_status;

/* flags (cualign_params.flags) */
#define CUALIGN_FLAG_DEVICE_PTRS      0x01u /* init arrays are device pointers */
#define CUALIGN_FLAG_EXACT            0x02u /* oracle-order fp64 sums: row sums of F in ascending f
                                               from 0.0, matching weight summed in ascending edge id
                                               (bitwise reproduces the oracle; slow on hub rows) */
#define CUALIGN_FLAG_OTHERMAX_LITERAL 0x04u /* reading Z4 literal: om(e) = max_{f!=e} v_f (no 0);
                                               default max-plus: om(e) = max(0, max_{f!=e} v_f) */
#define CUALIGN_FLAG_ROUND_DAMPED     0x08u /* reading Z5 variant: round y^p, z^p instead of y^c, z^c */
#define CUALIGN_FLAG_TIMING           0x10u /* record CUDA events around every kernel (diagnostics) */
#define CUALIGN_FLAG_MATCH_ROUNDS     0x20u /* a7 schedule: synchronous pointer rounds (paper's Phase 1/2)
                                               instead of the default Suitor proposals; same matching */
#define CUALIGN_FLAG_FP32_S           0x40u /* NEXT-3: store the square messages S^p (the dominant HBM
                                               stream, 16 -> 8 B per square) in fp32; all arithmetic
                                               stays fp64, S^p is rounded to fp32 on store.  Not an
                                               oracle reading: parity is to a tolerance (DESIGN.md
                                               "fp32 S^p"), not bitwise.  Rejected with EXACT. */

/* Undirected simple graph: symmetric CSR, row i lists the
 * neighbours of i strictly increasing, no self loops (reading Z14).
 * rowptr has n+1 entries, rowptr[0] = 0; col has rowptr[n] entries. */
typedef struct {
    int32_t n;
    const int64_t *rowptr;
    const int32_t *col;
} cualign_graph;

/* Candidate bipartite graph L = (V_A u V_B, E_L, w):
 * m edges (a[k], b[k]) with 0 <= a < n_A, 0 <= b < n_B, strictly increasing in
 * (a, b) lexicographic order -- the canonical edge id of (a[k], b[k]) is k --
 * and finite weights w[k]. */
typedef struct {
    int64_t m;
    const int32_t *a;
    const int32_t *b;
    const double *w;
} cualign_edges;

typedef struct {
    double alpha;     /* >= 0, weight of the matching term of Eq. 1 */
    double beta;      /* >= 0, weight of the overlap term of Eq. 1 */
    double gamma;     /* damping base, 0 < gamma <= 1; iteration p damps with
                         g = gamma^p, h = 1 - g computed on the host in fp64 (Z2) */
    uint32_t flags;   /* CUALIGN_FLAG_* */
    int32_t device;   /* CUDA device ordinal */
    void *stream;     /* cudaStream_t to run on (e.g. torch.cuda.current_stream());
                         NULL = the handle creates its own non-blocking stream */
    /* Sharding by contiguous A-vertex blocks (multi-GPU is the
     * paper's future work):
     *   world <= 1: one GPU, rank = 0, nccl_unique_id = NULL;
     *   world > 1, nccl_unique_id != NULL: this process is shard `rank` of
     *     `world` (one GPU each); init / iterate / round / run are collective
     *     over the ranks; the id comes from cualign_nccl_unique_id() on one
     *     rank, broadcast by the caller (e.g. torch.distributed);
     *   world > 1, nccl_unique_id == NULL, rank = -1: `world` virtual shards
     *     in this handle on one device, exchanging through device copies --
     *     the sharded path for single-GPU testing.
     * Results of a sharded run are bitwise those of world = 1.  Not with
     * CUALIGN_FLAG_EXACT. */
    int32_t rank;
    int32_t world;
    const void *nccl_unique_id; /* 128-byte ncclUniqueId or NULL */
    /* Result-neutral tuning (0 = automatic; every choice gives the same bits):
     *   schedule: step schedule of cualign_bp_run / run_trace with both
     *     halves of a step: 0 = chosen by the
     *     library, 1 = pipelined (rounding of iteration k beside iteration
     *     k+1), 2 = serial (iteration, then its rounding), 3 = forked (the
     *     rounding beside the square pass of its own iteration);
     *   square_tile_log: the squares are grouped into (e block, f block)
     *     tiles of 2^k edges; -1 = no tiles,
     *     1..30 = that block size. */
    int32_t schedule;
    int32_t square_tile_log;
} cualign_params;

/* Result of one rounding step (Alg. 2 l.17-24). */
typedef struct {
    int32_t iter;        /* BP iteration p the rounded messages belong to */
    int32_t source;      /* 0 = M_y chosen, 1 = M_z (M_y wins ties, reading Z8) */
    int32_t improved;    /* 1 if score > bestScore (strict) and best was replaced */
    int32_t best_iter;   /* iteration of the best matching so far (0 = none) */
    int32_t card_y, card_z;       /* |M_y|, |M_z| */
    double score_y, score_z;      /* alpha*w(M) + beta*overlap(M) */
    double weight_y, weight_z;    /* sum of the original w over M (reading Z9) */
    double score;                 /* max(score_y, score_z) */
    double best_score;            /* bestScore after this round (starts at 0) */
    int64_t overlap_y, overlap_z; /* x'Sx/2: squares {e,f} with both e, f in M */
    int32_t rounds_y, rounds_z;   /* matching work: successful proposals (Suitor schedule) or
                                     pointer rounds (CUALIGN_FLAG_MATCH_ROUNDS) */
} cualign_round_info;

/* Sizes of an initialised handle. */
typedef struct {
    int32_t n_a, n_b;
    int64_t m;          /* |E_L| */
    int64_t s;          /* nnz(S) = 2 * squares */
    int64_t squares;    /* s / 2 (reading Z18) */
    int64_t max_row;    /* longest S row */
    int32_t p;          /* iterations done */
    int32_t fixed_point_bits; /* fraction bits of the fast-mode F-sum accumulator */
    int64_t device_bytes;     /* device memory held by the handle */
    int32_t rank, world;      /* shard (rank -1 for a virtual-shard handle) */
    int64_t edge_begin, edge_end; /* owned canonical edge ids [begin, end) */
    int64_t squares_local;    /* squares stored by this shard */
    int32_t merge_rounds;     /* sharded rounding (NEXT-1): merge rounds of the last round() (0 if unsharded) */
    int32_t schedule;         /* step schedule run() selected: -1 not yet, 0 rounding forked beside the
                                 square pass, 1 pipelined (rounding of k beside iteration k+1), 2 serial */
} cualign_sizes;

/* Diagnostics: per-kernel-class event timing (needs CUALIGN_FLAG_TIMING) and
 * launch counts since the last reset. */
#define CUALIGN_NUM_KERNEL_CLASSES 10
typedef struct {
    int64_t launches;                              /* all kernels launched by the handle */
    int64_t class_launches[CUALIGN_NUM_KERNEL_CLASSES];
    double class_ms[CUALIGN_NUM_KERNEL_CLASSES];   /* summed event time */
    /* sharded handles: exchanges since the last reset */
    int64_t comm_calls;      /* exchange steps (a grouped set of collectives counts once) */
    int64_t comm_bytes_in;   /* bytes this process's shard(s) received (all-gathered,
                                reduced-to-owner or all-reduced data arriving from peers) */
    double comm_ms;          /* summed event time of the exchanges (timing on) */
} cualign_stats;
/* kernel classes */
#define CUALIGN_K_TOP2    0 /* a4: per-vertex top-2 of y^p (A rows) and z^p (B columns) */
#define CUALIGN_K_EDGE    1 /* a3 tail + a4 + a6 on vectors: d, y^c, z^c, u, damping of y, z */
#define CUALIGN_K_SQUARE  2 /* a3 + a5 + a6 on S values: the square pass (dominant kernel) */
#define CUALIGN_K_ROWSUM  3 /* exact mode: sequential row sums of F */
#define CUALIGN_K_MATCH   4 /* a7 + a8: matching on y^c and z^c, evaluate, best */
#define CUALIGN_K_INIT    5 /* a1 + a2: validation, L layouts, S build */
#define CUALIGN_K_STATE   6 /* get/set state gathers and scatters */
#define CUALIGN_K_OTHER   7 /* iteration counter advance */
#define CUALIGN_K_EVAL    8 /* a8: evaluate M_y, M_z + final score / select / best reduction */
#define CUALIGN_K_MATCHAUX 9 /* a7 bookkeeping: mates from suitors, best-matching copy */

/* a1 + a2: validate, copy A, B, L to the device, build L's A-side rows and
 * B-side incidence, build S (Alg. 3) and its square layout, zero the BP state
 * (Alg. 2 l.1-7).  n_A = A->n, n_B = B->n (reading Z15:
 * n_A != n_B allowed).  Validation failures return CUALIGN_EINVAL with a
 * message: out-of-range ids, unsorted or duplicate L edges, asymmetric graphs,
 * self loops, unsorted rows, non-finite w, alpha < 0, beta < 0,
 * gamma outside (0, 1].  On failure *out is set to NULL. */
cualign_status cualign_bp_init(const cualign_graph *A, const cualign_graph *B,
                               const cualign_edges *L, const cualign_params *params,
                               cualign_bp **out);

/* a3-a6: run n_steps iterations of Alg. 2 lines 9-16,
 * p += n_steps.  Asynchronous on the handle's stream.  n_steps >= 0. */
cualign_status cualign_bp_iterate(cualign_bp *h, int32_t n_steps);

/* a7-a8: Alg. 2 lines 17-24 on the current y^c, z^c: two matchings, evaluate,
 * select, best update -- all on the device.  info == NULL: fully asynchronous
 * (best is tracked on the device); otherwise synchronises and fills *info. */
cualign_status cualign_bp_round(cualign_bp *h, cualign_round_info *info);

/* a3-a8 repeated: n_steps x (iterate(1) if what & CUALIGN_RUN_ITERATE, then
 * round if what & CUALIGN_RUN_ROUND), replayed from a CUDA graph of one step
 * captured on first use (no host work per kernel; g = gamma^p is read by the
 * kernels from a host-computed table, reading Z2).  Same results as the
 * equivalent sequence of iterate/round calls.  Asynchronous on params.stream;
 * read results with get_best.  what must be 1, 2 or 3. */
#define CUALIGN_RUN_ITERATE 1
#define CUALIGN_RUN_ROUND   2
cualign_status cualign_bp_run(cualign_bp *h, int32_t n_steps, int32_t what);

/* End-to-end loop of Alg. 2: n_steps x (iterate(1) +
 * round), as cualign_bp_run(h, n_steps, CUALIGN_RUN_ITERATE |
 * CUALIGN_RUN_ROUND), and infos[k] (host array of n_steps, caller-owned)
 * receives the round info of step k with best_score / best_iter as of that
 * step.  Each step's info is copied to the host as soon as its rounding has
 * finished (stream-ordered, into pinned staging), so the host never stalls the
 * device between steps; synchronises once before returning.  Errors: EINVAL
 * for n_steps < 0 or a NULL infos with n_steps > 0. */
cualign_status cualign_bp_run_trace(cualign_bp *h, int32_t n_steps, cualign_round_info *infos);

/* Diagnostics: enable (1) / disable (0) per-kernel event timing (as
 * CUALIGN_FLAG_TIMING).  Graph replays with timing on synchronise after each
 * step to read the per-kernel events; results via cualign_bp_get_stats. */
cualign_status cualign_bp_set_timing(cualign_bp *h, int32_t on);

/* Best matching so far: mate_a[a] = canonical id of the L edge matched at A
 * vertex a, or -1 (host buffer of n_A int32; may be NULL).  info receives the
 * last round's info with best_score / best_iter (may be NULL). Synchronises. */
cualign_status cualign_bp_get_best(cualign_bp *h, int32_t *mate_a, cualign_round_info *info);

/* Release everything; NULL-safe. */
void cualign_bp_free(cualign_bp *h);

/* Sizes of the problem (m, s, ...).  Synchronises. */
cualign_status cualign_bp_get_sizes(cualign_bp *h, cualign_sizes *sizes);

/* S in CSR form over canonical edge ids (row e lists f ascending):
 * rowptr (m+1 int64), col (s int32); either may be NULL; *s_out = nnz(S). */
cualign_status cualign_bp_get_S(cualign_bp *h, int64_t *rowptr, int32_t *col, int64_t *s_out);

/* State after the last iterate (host buffers, each may be NULL):
 * yc, zc, yp, zp, d: m doubles; Sp: s doubles in get_S's CSR order; p: int.
 * Sharded handles: Sp must be NULL; a virtual-shard handle assembles the
 * owners' slices, a process shard returns arrays whose owned slice
 * [edge_begin, edge_end) is valid (rounding is sharded too, NEXT-1, so the
 * messages are never all-gathered). */
cualign_status cualign_bp_get_state(cualign_bp *h, double *yc, double *zc, double *yp,
                                    double *zp, double *d, double *Sp, int32_t *p);

/* Inject (y^p, z^p, S^p, p) (host buffers: m, m, s doubles in CSR order) --
 * checkpoint/resume and one-step parity.  The next iterate runs iteration p+1. */
cualign_status cualign_bp_set_state(cualign_bp *h, const double *yp, const double *zp,
                                    const double *Sp, int32_t p);

/* The two matchings of the last rounding (Alg. 2 l.17-20):
 * mate_y[a] / mate_z[a] = canonical id of the L edge matched at A vertex a in
 * M_y (rounding of y^c, or y^p with CUALIGN_FLAG_ROUND_DAMPED) / M_z, or -1
 * (host buffers of n_A int32; either may be NULL).  Sharded handles: the
 * replicated final matchings.  ESTATE before the first rounding.
 * Synchronises. */
cualign_status cualign_bp_get_round_mates(cualign_bp *h, int32_t *mate_y, int32_t *mate_z);

/* Sampled S^p (test / diagnostic hook for one-step parity at sizes where the
 * full S^p does not fit the host): every square {e, f} (e < f, S_ef = S_fe =
 * 1) with e or f in edges[0..n) (host array of canonical ids),
 * as e_out[i] = e, f_out[i] = f, v_ef[i] = S^p_ef, v_fe[i] = S^p_fe (host
 * buffers of cap entries; any may be NULL), in unspecified order.  At most cap
 * are written; *n_out receives the number of such squares (call again with a
 * larger cap if it exceeds cap).  Single-GPU and virtual-shard handles (a
 * process shard holds only its own squares: ESTATE).  EINVAL on an id
 * outside [0, m).  Synchronises. */
cualign_status cualign_bp_sample_squares(cualign_bp *h, const int32_t *edges, int64_t n, int64_t cap,
                                         int32_t *e_out, int32_t *f_out, double *v_ef, double *v_fe,
                                         int64_t *n_out);

/* Diagnostics; reset = 1 clears counters after reading. Synchronises. */
cualign_status cualign_bp_get_stats(cualign_bp *h, cualign_stats *stats, int32_t reset);

/* a7 standalone: the locally-dominant 1/2-approximate matching of L weighted by
 * x (m doubles; host, or device if CUALIGN_FLAG_DEVICE_PTRS) with the strict
 * order (x desc, edge id asc), only x > 0 eligible (readings Z6, Z7).  Writes
 * mate_a (n_A int32) and mate_b (n_B int32) host buffers (either may be NULL):
 * the matched edge id at each vertex or -1.  *rounds_out (may be NULL)
 * receives the matching work (see cualign_round_info.rounds_y).  L->w is
 * ignored (may be NULL). */
cualign_status cualign_match(const cualign_edges *L, int32_t n_a, int32_t n_b, const double *x,
                             const cualign_params *params, int32_t *mate_a, int32_t *mate_b,
                             int32_t *rounds_out);

/* NEXT-4 quality harness: scores of an alignment of A to B against the
 * network-alignment quality measures the paper uses (PAPER.md:327-333,
 * "NCV-GS^3 ... normalized by the sizes of the networks", defined in its
 * refs [18, 20]):
 *   conserved = A edges {i, j} with {M(i), M(j)} in E_B  (= overlap, :60)
 *   induced   = B edges with both ends in M(V_A)
 *   NC   = correct / truth_total          (node correctness vs the ground truth P, :327)
 *   EC   = conserved / |E_A|              (edge correctness)
 *   ICS  = conserved / induced            (induced conserved structure)
 *   S3   = conserved / (|E_A| + induced - conserved)   (symmetric substructure score)
 *   NCV  = 2 aligned / (|V_A| + |V_B|)    (node coverage)
 *   GS3  = S3 (one-to-one alignment)
 *   NCV-GS3 = sqrt(NCV * GS3)
 * A ratio with a zero denominator is 0. */
typedef struct {
    int64_t n_a, n_b;         /* |V_A|, |V_B| */
    int64_t edges_a, edges_b; /* undirected edge counts */
    int64_t aligned;          /* A vertices with an image */
    int64_t truth_total;      /* A vertices with a true image (0 without truth) */
    int64_t correct;          /* A vertices mapped to their true image */
    int64_t conserved;
    int64_t induced;
    double nc, ec, ics, s3, ncv, gs3, ncv_gs3;
} cualign_quality;

/* Evaluate the alignment map_ab (n_A int32: B vertex of each A vertex, -1 =
 * unaligned; must be injective) against A, B (validated like
 * cualign_bp_init) and the optional ground truth (n_A int32, -1 = none; NULL
 * = no truth).  Pointers are host pointers unless CUALIGN_FLAG_DEVICE_PTRS;
 * params supplies flags / device / stream only.  EINVAL on a map entry out
 * of range or two A vertices mapped to one B vertex. */
cualign_status cualign_quality_eval(const cualign_graph *A, const cualign_graph *B, const int32_t *map_ab,
                                    const int32_t *truth, const cualign_params *params,
                                    cualign_quality *out);

/* NEXT-2: kNN sparsification -- L from given embeddings, Alg. 1 lines 7-14
 * (PAPER.md:133-140, :121): s(u, v) = cosine similarity of Y_A(u) and Y_B(v)
 * (l.9) for all pairs, and for every A vertex the k most similar B vertices
 * (reading Z19; ties to the lower B index).  YA (n_a x d) and YB (n_b x d) are
 * row-major fp32 (host, or device with CUDA_FLAG_DEVICE_PTRS), 1 <= d <= 256,
 * 1 <= k <= min(32, n_b), all entries finite (EINVAL otherwise).  A zero row
 * has similarity 0 with everything.  Writes m = n_a * k edges into the
 * caller's L_a, L_b (int32) and L_w (double, the similarity) in canonical
 * order (a ascending, then b ascending) -- ready for cualign_bp_init.
 * Precision: tensor-core products of the unit rows rounded to bf16, fp32
 * accumulation. */
cualign_status cualign_knn(const float *YA, int32_t n_a, const float *YB, int32_t n_b, int32_t d, int32_t k,
                           const cualign_params *params, int32_t *L_a, int32_t *L_b, double *L_w);

/* NCCL unique id for a sharded init (write len >= 128 bytes into id). */
cualign_status cualign_nccl_unique_id(void *id, int32_t len);

/* Message of the last failing call on this thread ("" if none). */
const char *cualign_last_error(void);

/* Library version string. */
const char *cualign_version(void);

#ifdef __cplusplus
}
#endif

#endif /* CUALIGN_BP_H */
