/*
 * mce.h -- C ABI of the B200-native maximum clique engine
 *          (libmce_b200.so, built from paper_conf_ipps_geilpo23_b200/csrc).
 *
 * Problem statement (Sec. II, line 47): for an undirected simple
 * graph G = (V, E), find omega(G) -- the size of the largest clique --, its
 * multiplicity (the number of cliques of size omega), and the members of
 * every clique of size omega ("enumeration", Sec. I line 35), or a single
 * maximum clique ("windowed search ... for finding a single, maximum clique
 * when memory constraints prevent enumeration", Sec. I line 40 and IV-E).
 *
 * Conventions shared by every call:
 *  - Vertices are 0..n-1 (int32 ids, n < 2^31).  The graph is given as CSR
 *    with BOTH directions of every undirected edge stored, each adjacency list
 *    sorted ascending, no self loops, no duplicates (PAPER.md V line 235:
 *    "ensure all graphs are undirected and contain no loops").  Violations are
 *    reported as MCE_ERR_INVALID by mce_load_csr when `validate` is set.
 *  - Every call returns an mce_status; on failure mce_last_error() returns a
 *    thread-local, NUL-terminated description (owned by the library).
 *  - `stream` is a cudaStream_t (may be NULL = legacy default stream).  Calls
 *    are synchronous with respect to the host on return unless stated.
 *  - Pointers marked (device) must be device-accessible memory of the handle's
 *    device; (host) pointers must be host memory.  The library never takes
 *    ownership of caller memory.
 *  - No CPU fallback exists: without a usable sm_100 device every call that
 *    needs the GPU fails with MCE_ERR_CUDA.
 */
#ifndef MCE_B200_H
#define MCE_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    MCE_OK = 0,
    MCE_ERR_INVALID = 1,  /* bad argument or malformed graph */
    MCE_ERR_CUDA = 2,     /* CUDA runtime error (incl. no device) */
    MCE_ERR_NOMEM = 3,    /* device allocation failed */
    MCE_ERR_BUDGET = 4,   /* a single frontier entry set cannot fit the memory budget */
    MCE_ERR_STATE = 5,    /* call out of order (e.g. result already fetched) */
    MCE_ERR_SYNC = 6      /* the bound_sync callback reported a failure (negative return) */
} mce_status;

typedef struct mce_graph mce_graph;   /* device-resident graph + preprocessing */
typedef struct mce_result mce_result; /* omega, multiplicity, cliques */

enum { MCE_WHERE_HOST = 0, MCE_WHERE_DEVICE = 1 };

/* Vertex ordering used to orient edges (PAPER.md IV-C line 131: "we use only
 * one of the two directed edges that represent each undirected edge"). */
enum { MCE_ORIENT_DEGENERACY = 0,     /* k-core peel order (north star); the asynchronous
                                         peel's order within a level depends on timing */
       MCE_ORIENT_DEGREE = 1,         /* (degree, id) order (the paper's choice) */
       MCE_ORIENT_DEGENERACY_DET = 2  /* a degeneracy order that is a function of the graph
                                         alone: (core, synchronous round of the peel of the
                                         core's shell, id); every process computes the same
                                         one (multi-GPU sharding, no broadcast) */ };

/* Greedy heuristic for the initial lower bound (PAPER.md IV-A, Table I). */
enum { MCE_HEUR_NONE = 0,
       MCE_HEUR_SINGLE_DEGREE = 1, MCE_HEUR_SINGLE_CORE = 2,
       MCE_HEUR_MULTI_DEGREE = 3, MCE_HEUR_MULTI_CORE = 4 };

/* Upper bound used to prune a candidate (C, P) (PAPER.md II-B-3, line 63). */
enum { MCE_BOUND_SIZE = 0,    /* |C| + |P|                         */
       MCE_BOUND_COLOR = 1 }; /* |C| + #colours of greedy colouring of P */

typedef struct {
    int32_t orientation;     /* MCE_ORIENT_* */
    int32_t heuristic;       /* MCE_HEUR_* */
    int64_t heuristic_runs;  /* h for the multi-run heuristics; <=0 means |V| */
    int32_t bound;           /* MCE_BOUND_* */
    int32_t lower_bound;     /* extra known lower bound on omega (0 = none) */
    int64_t window;          /* roots per window (PAPER.md IV-E); <=0 = all roots at once */
    int64_t budget_bytes;    /* device bytes the frontier may use; <=0 = half of the free device
                                memory.  Allocated on demand in segments (the first sized
                                ~1 GiB + 48 B/edge), kept on the graph for later calls. */
    int64_t max_cliques;     /* capacity of the stored clique list; <=0 = unbounded
                                (still limited: at most max(2^20, rows fitting a quarter
                                of the budget) are stored).  The multiplicity is
                                always exact; cliques beyond capacity are counted
                                but not stored (mce_result_info: truncated). */
    int32_t shard_rank;      /* root sharding for multi-GPU: this process takes the */
    int32_t shard_count;     /*   roots with index % shard_count == shard_rank (<=1: all) */
    /* Optional per-step bound exchange (multi-GPU).  Called after every
     * expansion step with this shard's best clique size and whether it still
     * has work; must return the global best (>= 0) and set *global_active to 1
     * while any shard has work.  Shards call it a DIFFERENT number of times
     * (one call per level / window / chunk of their own work): the exchange
     * is a collective that pairs the k-th calls of all shards, whatever step
     * each is at; a shard that has finished keeps calling it with
     * local_active = 0 until *global_active comes back 0, so every shard
     * leaves in the same collective round.  A negative return means the
     * exchange failed (e.g. a peer is gone): the call stops with
     * MCE_ERR_SYNC.  The returned bound only ever raises the pruning bound to
     * a size some shard has found, so the pairing does not affect results. */
    int32_t (*bound_sync)(int32_t local_best, int32_t local_active, int32_t *global_active, void *user);
    void *bound_sync_user;
    int32_t verbose;         /* >0: per-level statistics on stderr */
    int32_t legacy_roots;    /* 0 (default): roots with |N+(r)| <= 64 take the fused root-level
                                kernel (adjacency build + first expansion in one warp, only
                                surviving roots materialised); 1: the generic per-level path
                                for every root (kept for A/B parity tests) */
    int32_t no_fused_levels; /* 0 (default): consecutive levels of at most 1024 candidates (<= 256
                                bits each) run inside one launch (expand_small); 1: every
                                level takes the count -> scan -> write launches (A/B tests) */
    int32_t no_clique_shortcut; /* 0 (default, colouring bound only): a candidate (C, P) whose P is
                                itself a clique with |C| + |P| equal to the size sought is
                                recorded as the clique C + P instead of being expanded level by
                                level (its only clique of that size; reading 10);
                                1: Algorithm 2's expansion of every level (A/B tests) */
    int32_t no_fused_expand; /* 0 (default): a level's count pass also writes the children (slots
                                reserved per warp, colouring computed once) whenever they fit half
                                of the free budget; 1: count -> scan -> write passes (A/B tests) */
    int32_t shard_depth;     /* with shard_count > 1: <= 1 (default): roots are dealt to shards by CSR
                                id; d >= 2: every shard expands all roots through level d - 1 and
                                keeps the level-d candidates (d-cliques) whose vertex-path hash
                                % shard_count == shard_rank (balances work that sits under a few
                                hub roots); cliques found above level d (leaves: clique /
                                pair completions are off above the split, their firing
                                depends on the shard's bound) are reported by shard 0 */
    int32_t no_overlap;      /* 0 (default): the degree heuristics run on a second stream and host
                                thread while the k-core / orientation preprocessing runs (they
                                share no data); 1: one after the other */
    int32_t no_reroot;       /* 0 (default): candidates of levels >= 2 at least MCE_REROOT_MIN_W
                                words wide (environment; unset = never, the measured best: on
                                R-MAT scale 26 the re-root matrix builds cost more than the
                                narrower expansion saves) become roots of their own over their
                                candidate set P (at the width of |P|); 1: never (A/B tests) */
    int32_t no_smem_expand;  /* 0 (default): levels of 8 or 16 words per candidate set are grouped by
                                root and expanded with the root's adjacency matrix staged in
                                shared memory (expand_smem); 1: rows read from global memory
                                (expand_tile; A/B tests) */
    int32_t no_root_colour;  /* 0 (default, colouring bound only): when many vertices can be in a
                                clique of the size sought (core >= need - 1, PAPER.md II-B-2), they
                                are greedily coloured once in reverse degeneracy order on the device
                                and a root whose out-neighbourhood meets fewer than need - 1
                                colours is dropped before its adjacency matrix is built (a proper
                                colouring of G restricted to N+(r) bounds every clique there;
                                DESIGN.md reading 14); 1: off (A/B tests) */
} mce_options;

/* Fill `opt` with defaults: degeneracy orientation, multi-run degree heuristic
 * with h = |V| (PAPER.md V-B-4: "The best default choice for an unknown
 * dataset is the multi-run degree heuristic"), colouring bound, no window,
 * 90% of free memory, unbounded clique list, no sharding. */
void mce_default_options(mce_options *opt);

/* Load a graph onto `device` (PAPER.md IV line 99: "convert the input dataset
 * into CSR format, which we store in GPU global memory").
 *   n        : number of vertices (>= 0)
 *   row_ptr  : int64[n+1], row_ptr[0] = 0, row_ptr[n] = nnz = 2|E|
 *   col_idx  : int32[nnz]
 *   where    : MCE_WHERE_HOST (copied to the device) or MCE_WHERE_DEVICE
 *              (copied device-to-device; the caller keeps its buffers)
 *   validate : nonzero = check symmetry/sortedness/no loops on the device
 * On success *out owns a device copy of the CSR; free with mce_graph_free. */
mce_status mce_load_csr(int32_t device, int64_t n, const int64_t *row_ptr, const int32_t *col_idx,
                        int32_t where, int32_t validate, void *stream, mce_graph **out);

void mce_graph_free(mce_graph *g);

/* Drop the cached preprocessing (core numbers, orientation) so that the next
 * mce_enumerate / mce_find_one recomputes it -- used by benchmarks that time
 * the whole pipeline from a resident CSR. */
mce_status mce_graph_clear_cache(mce_graph *g);

/* k-core decomposition + orientation (PAPER.md II-B-2 line 61, IV-C line
 * 131).  Run implicitly by mce_enumerate / mce_find_one; exposed for tests.
 * core_out (device or host per `where`, int32[n], may be NULL): core numbers.
 * order_out (int32[n], may be NULL): vertex of rank i (the orientation order;
 * every edge points from lower to higher rank).  *degeneracy_out = max core. */
mce_status mce_preprocess(mce_graph *g, int32_t orientation, int32_t *core_out, int32_t *order_out,
                          int32_t where, int32_t *degeneracy_out);

/* Replace the orientation order with `order` (int32[n], a permutation of the
 * vertices: vertex of rank i; host or device per `where`) and rebuild the
 * oriented CSR from it; core numbers are computed if missing.  Multi-GPU:
 * the k-core peel order is not deterministic across processes and root /
 * candidate sharding needs every rank to orient edges the same way, so
 * rank 0's order is broadcast and set on the others (distributed.py).  For
 * MCE_ORIENT_DEGENERACY the order must be a degeneracy order (each vertex
 * has at most core(v) later neighbours) -- e.g. another rank's
 * mce_preprocess output; MCE_ERR_INVALID for a NULL order. */
mce_status mce_set_order(mce_graph *g, int32_t orientation, const int32_t *order, int32_t where);

/* Install k-core numbers and a degeneracy (peel) order computed elsewhere
 * instead of peeling on this handle (PAPER.md IV-C: the degeneracy ordering
 * and core numbers of the preprocessing step).  core: int32[n], core number of
 * each vertex; peel: int32[n], vertex of rank i in a degeneracy order (each
 * vertex has at most core(v) later neighbours) -- both host or device per
 * `where`, copied, caller keeps ownership.  Not validated: they must be exact
 * (e.g. another handle's mce_preprocess(MCE_ORIENT_DEGENERACY) output on the
 * same graph).  The handle's orientation is dropped and rebuilt from them on
 * the next call; the degeneracy is recomputed as max core.  Multi-GPU: rank 0
 * peels, broadcasts both arrays and the other ranks set them here, so every
 * rank orients the edges the same way without a second (or a deterministic,
 * slower) peel (distributed.py).  MCE_ERR_INVALID for NULL arrays (n > 0). */
mce_status mce_set_core(mce_graph *g, const int32_t *core, const int32_t *peel, int32_t where);

/* Greedy heuristic (PAPER.md IV-A, Algorithm 1).  kind = MCE_HEUR_*; h = runs
 * (<=0: |V|; single-run kinds ignore h and use 1).  *omega_bar_out = size of the
 * best clique found; clique_out (host, capacity >= max degree + 1, may be NULL)
 * receives that clique (original vertex ids, in the order added) and
 * *clique_len_out its length.  run_size_out (host int32[h], may be NULL): size of
 * run i where seeds are ordered by (threshold desc, id asc). */
mce_status mce_heuristic(mce_graph *g, int32_t kind, int64_t h, int32_t *omega_bar_out, int32_t *clique_out,
                         int32_t *clique_len_out, int32_t *run_size_out);

/* Enumerate every maximum clique (PAPER.md IV-D, Algorithm 2, breadth-first).
 * On success *out holds omega, the multiplicity and the cliques.  Work is
 * ordered on `stream` (mce_load_csr); the overlapped heuristic uses a second,
 * library-owned stream that waits on `stream` and is joined before return.
 * Errors: MCE_ERR_BUDGET when one candidate's children exceed the frontier
 * budget, MCE_ERR_CUDA / MCE_ERR_NOMEM from the runtime; *out is NULL then. */
mce_status mce_enumerate(mce_graph *g, const mce_options *opt, mce_result **out);

/* Find one maximum clique with the windowed search (PAPER.md IV-E): roots are
 * processed `window` at a time (opt->window overrides when > 0) and the lower
 * bound is raised after every window.  The result holds omega, multiplicity 1
 * and one clique of size omega. */
mce_status mce_find_one(mce_graph *g, int64_t window, const mce_options *opt, mce_result **out);

/* Result accessors.  omega: clique number; count: multiplicity (exact);
 * stored: cliques available to fetch (< count only when truncated). */
mce_status mce_result_info(const mce_result *r, int32_t *omega, int64_t *count, int64_t *stored,
                           int32_t *truncated);
/* Copy the stored cliques, each sorted ascending, the list in lexicographic
 * order, as int32[stored * omega] into dst (host or device per `where`).
 * The canonical rows stay in device memory owned by the result until this
 * call copies them (one device-to-host or device-to-device copy). */
mce_status mce_result_cliques(mce_result *r, int32_t *dst, int32_t where);
/* Per-level statistics of the last run: entries[k] = candidates (C, P) with
 * |C| = k+1 that were expanded, for k < levels (host int64 array of capacity
 * `cap`).  *levels_out = number of levels recorded. */
mce_status mce_result_levels(const mce_result *r, int64_t *entries, int32_t cap, int32_t *levels_out);
/* Kernel timing of the last run, milliseconds measured with CUDA events on
 * the run's stream: [0] preprocess, [1] heuristic ([0] and [1] overlap when
 * the degree heuristic runs on the library's second stream, mce_options.no_overlap),
 * [2] expansion total,
 * [3] dominant expansion kernel total, [4] number of dominant-kernel launches,
 * [5] algorithmic bytes moved by the dominant kernel, [6] kernels launched,
 * [7] fused root-level kernel total, [8] its launches, [9] its algorithmic
 * bytes (16 + 20 L + 4 T per root: row bounds, V, and the out-rows of V),
 * [10] host wall time of the whole call, [11] of its preprocessing, [12] of
 * its heuristic, [13] host<->device synchronisations it made, [14] host
 * time of the budget / workspace setup, [15] of the root classes + levels,
 * [16] of the canonical read-out of the stored cliques (device sort + copy),
 * [17] device time of the root setup: root colour filter and the root /
 * re-root adjacency matrix builds (not part of [2]), [18] of the root matrix
 * builds alone (build_adj_block), [19] their launches, [20] their
 * algorithmic bytes (V and row bounds 20 B per member, every out-row id the
 * scan reads 4 B, the matrix 8 W B per row). */
mce_status mce_result_timing(const mce_result *r, double *t, int32_t cap);
void mce_result_free(mce_result *r);

/* Device memory freed by the library (graph handles, regrown workspaces) is
 * cached per device and reused by later calls, so a new graph or a new call
 * does not pay cudaMalloc/cudaFree.  This returns the cached blocks of
 * `device` to the driver.  MCE_ERR_INVALID for a bad device index. */
mce_status mce_empty_cache(int32_t device);

const char *mce_last_error(void);
const char *mce_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MCE_B200_H */
