/*
 * dbc.h -- C ABI of the B200 dynamic betweenness-centrality library (libdbc.so).
 *
 * Method: McLaughlin & Bader, "Revisiting Edge and Node Parallelism for Dynamic
 * GPU Graph Analytics".  Citations are "P:<line>" into
 * /root/reference/PAPER.md, plus the section / algorithm / equation.
 *
 *  - The library stores, for each root s of a root set R, the BFS distance
 *    d_s(t), the shortest-path count sigma_st and the dependency delta_s(t) for
 *    every vertex t (Sec. II-D), and the betweenness partial
 *    BC(v) = sum_{s in R, s != v} delta_s(v) (Eq. (3); ordered pairs,
 *    unscaled -- DESIGN.md reading R1).
 *  - dbc_static_compute runs Brandes' algorithm (Alg. 1) over the
 *    local roots: it builds the state and is the GPU recompute baseline
 *    (Table III).
 *  - dbc_insert_edges applies edge insertions one at a time (Sec. IV):
 *    for every root the insertion is classified by d_s(u) vs d_s(v) (Cases 1/2/3,
 *    P:148-159); affected vertices get d/sigma repaired by a frontier-queued
 *    forward pass (Alg. 2 stage 2 / Alg. 5) and delta/BC by a
 *    reverse level-ordered pass (Alg. 2 stage 3 / Alg. 7 / Alg. 8, P:198-240,
 *    P:366-432).  The result equals a recompute from scratch on the new graph.
 *
 * Conventions shared by every call
 *  - Every call returns dbc_status (0 = DBC_OK, < 0 = error).  No exception,
 *    abort or exit crosses the ABI.  On error, dbc_last_error(ctx) holds a
 *    one-line message and the context state is unchanged unless stated.
 *  - Vertices are int32 in [0, n).  Unreachable: d = DBC_INF (INT32_MAX),
 *    sigma = 0, delta = 0.  delta_s(s) = 0 by convention.
 *  - Host pointers are borrowed for the duration of the call only (copied).
 *    Device pointers (suffix _device) must be device memory of opt->device and
 *    must stay valid until the work enqueued by the call has completed on the
 *    context stream.
 *  - All device work runs on one CUDA stream (opt->stream, or a stream the
 *    library creates).  Calls returning host data synchronise that stream.
 *  - A context is not thread-safe.  Several contexts may coexist (e.g. one per
 *    GPU and rank).
 *  - Multi-GPU: every rank passes the FULL root list; rank r owns root slots
 *    with slot % world == r.  The per-rank BC partials
 *    are summed across ranks -- the only cross-GPU exchange of the method
 *     -- by dbc_get_bc itself, through the context's own NCCL
 *    communicator (opt->nccl_id) or the caller's reduction callback
 *    (opt->reduce); dbc_get_bc_partial_device exposes the partial for callers
 *    that reduce it themselves.
 */
#ifndef DBC_H
#define DBC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DBC_INF INT32_MAX
#define DBC_ABI_VERSION 2

typedef struct dbc_ctx dbc_ctx; /* opaque; owns all device memory it allocates */

typedef enum {
    DBC_OK = 0,
    DBC_EINVAL = -1,     /* bad argument (NULL, n < 1, bad CSR, bad slot, ...) */
    DBC_ENOMEM = -2,     /* device or host allocation failed */
    DBC_ECUDA = -3,      /* CUDA runtime error (message in dbc_last_error) */
    DBC_ENCCL = -4,      /* NCCL missing or a collective failed (message in dbc_last_error) */
    DBC_ESTATE = -5,     /* call out of order, e.g. insert before static_compute */
    DBC_EEDGE = -6,      /* self loop, out-of-range vertex, edge already present,
                            or duplicate edge within a batch; batch not applied */
    DBC_ECAPACITY = -7,  /* inserted-edge capacity (opt.edge_capacity) exhausted */
    DBC_ENUMERIC = -8    /* a shortest-path count overflowed fp64 to +inf */
} dbc_status;

/* Flags for dbc_options.flags */
#define DBC_FLAG_MODE_S   0x1u /* one update launch per insertion (paper structure,
                                  P:244-252); default is the root-asynchronous
                                  batch kernel (Mode A, one launch per batch).
                                  Both give identical d/sigma.                     */
#define DBC_FLAG_TIMING   0x2u /* record CUDA events around the library's kernels;
                                  read with dbc_get_timings                        */
#define DBC_FLAG_EXACT_BC 0x4u /* dbc_get_bc / dbc_get_bc_partial_device rebase the
                                  partial as sum over local slots of delta_s(v)
                                  (Eq. (3)) instead of the incrementally updated
                                  value: removes drift over long streams          */
#define DBC_FLAG_NO_REORDER 0x8u /* keep the caller's vertex numbering internally
                                  (default: BFS-order relabelling for locality;
                                  invisible at the ABI, results identical)        */
#define DBC_FLAG_NO_MERGE 0x10u /* Mode A: one job per (root, insertion), the
                                  paper's one-at-a-time structure.
                                  Default: each root repairs a window of up to
                                  16384 insertions of the batch as ONE job seeded
                                  with every endpoint pair (R18): d and
                                  sigma after the batch are bit-identical, BC
                                  within rounding (the sum of the per-insertion
                                  changes telescopes)                            */

#define DBC_FLAG_PULL_DELTA 0x40u /* debug mode: every vertex the update touches
                                  (Alg. 2's t[v] != untouched) recomputes
                                  delta by the pull of Eq. (2) in canonical order
                                  instead of the push-delta form (SURVEY.md Sec.
                                  8(c) item 14), and the static pass sums long
                                  rows in canonical order too: delta is then
                                  bit-identical to the oracle, and with
                                  DBC_FLAG_EXACT_BC at world 1 so is BC.  Every
                                  batch runs one job per insertion.  Not with
                                  deletions or DBC_FLAG_EDGE_PARALLEL (EINVAL) */

#define DBC_FLAG_EDGE_PARALLEL 0x20u /* edge-based parallel update (Alg. 4 / Alg. 6,
                                  P:278-356): one launch per insertion, every
                                  level a pass of one CTA per root over all
                                  edges -- the comparison kernel of Table II
                                  (P:458-478).  Same results as the default
                                  node-based kernel; slower by design        */

/* Sum all-reduce of the BC partial across ranks, in place: bc_device is
 * fp64[n] device memory of the context's device, stream its CUDA stream (the
 * reduction must be complete, or ordered on that stream, when the callback
 * returns).  Return 0 on success; anything else makes dbc_get_bc fail with
 * DBC_ENCCL. */
typedef int (*dbc_reduce_fn)(double *bc_device, int64_t n, void *stream, void *user);
/* Device memory hooks (e.g. torch's caching allocator): return NULL on failure. */
typedef void *(*dbc_alloc_fn)(size_t bytes, void *user);
typedef void (*dbc_free_fn)(void *ptr, void *user);

/* Tuning of the kernels' launch configuration.  Results
 * never depend on it.  dbc_tuning_default sets every field to "automatic"
 * (integers < 0, heavy_factor 0, disable 0); the automatic choices are the
 * ones measured best on B200. */
typedef struct {
    int32_t update_block;    /* batch kernel CTA width: 128, 256, 512 or 1024            */
    int32_t update_pair;     /* 512-thread batch CTAs built for two per SM: 0 / 1        */
    int32_t static_block;    /* static Brandes CTA width: 128, 256, 512 or 1024          */
    int32_t window;          /* insertions merged into one job per root (R18)  */
    int32_t heavy_cap;       /* roots run on the wide heavy lane per batch (0: none)     */
    float heavy_factor;      /* a root is heavy if its last chain took > this x median   */
    int32_t help_down_min;   /* batch kernel: down levels of >= this many items are helped */
    int32_t help_down_block; /* ... in blocks of this many items                         */
    int32_t help_entries;    /* flattened passes: entries per help block                 */
    int32_t help_min_blocks; /* ... published from this many blocks                      */
    int32_t busy_help;       /* blocks a busy worker takes at a level boundary (0: none) */
    int32_t busy_min;        /* ... of passes of at least this many blocks               */
    int32_t down_long_min;   /* entry-balanced long rows of a down level from this many entries */
    int32_t wide_inlane;     /* up levels of <= this many items per thread: short rows in-lane */
    int32_t lean_block;      /* per-insertion kernel CTA width: 128, 256, 512 or 1024    */
    int32_t lean_workers;    /* its worker CTAs (capped at the resident maximum)         */
    int32_t lean_max_batch;  /* merged batches of <= this many insertions run per insertion */
    int32_t lean_short;      /* level-2 rows longer than this x deg(root) probe adj(root) */
    int32_t trace_slot;      /* -DDBC_PHASE_TIMERS builds: trace this root slot          */
    uint32_t disable;        /* DBC_TUNE_* bits                                          */
    int32_t static_ms;       /* static Brandes: 1 multi-source (32 roots per warp), 0 one
                                root per CTA; automatic: multi-source on graphs of mean
                                degree >= 8 (falls back to per-root when a BFS passes
                                level 254 or its level lists overflow)                  */
    int32_t static_groups;   /* multi-source: 32-root groups traversed together          */
    int32_t static_chunk;    /* multi-source: row entries per warp task                  */
    int32_t static_width;    /* multi-source: roots per group, 32 or 64 (two per lane)   */
    uint32_t reserved[4];    /* must be zero                                             */
} dbc_tuning;
#define DBC_TUNE_NO_HELP      0x1u  /* batch kernel: no cooperative help          */
#define DBC_TUNE_NO_HEAVY     0x2u  /* batch kernel: no heavy lane                */
#define DBC_TUNE_NO_LEAN      0x4u  /* per-insertion jobs on the batch kernel     */
#define DBC_TUNE_NO_LEAN_HELP 0x8u  /* per-insertion kernel: no cooperative help  */
#define DBC_TUNE_NO_LOWDEG    0x10u /* batch kernel: no in-lane up levels on low-degree graphs */

typedef struct {
    int32_t device;        /* CUDA device ordinal (default 0)                      */
    int32_t rank;          /* this process's rank in [0, world) (default 0)        */
    int32_t world;         /* number of ranks / GPUs sharing the root set (def. 1) */
    int32_t workers;       /* persistent worker CTAs; 0 = automatic                */
    int64_t edge_capacity; /* max undirected edges inserted over the context's
                              lifetime; 0 = automatic (max(2^16, m/4))            */
    void *stream;          /* cudaStream_t to run on; NULL = library-owned stream;
                              cudaStreamLegacy ((void*)1) = the legacy default stream */
    uint32_t flags;        /* DBC_FLAG_*                                           */
    uint32_t pad0;         /* must be zero                                         */
    const dbc_tuning *tuning;  /* nullable: automatic; copied by dbc_create        */
    const void *nccl_id;   /* nullable: 128-byte ncclUniqueId (dbc_nccl_unique_id on
                              rank 0, shared with every rank).  dbc_create then
                              joins an NCCL communicator of `world` ranks (a
                              collective call: every rank must create) that
                              dbc_get_bc uses for the BC all-reduce over NVLink  */
    dbc_reduce_fn reduce;  /* nullable: the BC all-reduce as a callback instead   */
    void *reduce_user;
    dbc_alloc_fn dev_alloc;  /* nullable: device allocations through the caller    */
    dbc_free_fn dev_free;    /* (both or neither)                                  */
    void *alloc_user;
    uint32_t reserved[4];  /* must be zero                                         */
} dbc_options;

/* Per-call counters.  Filled when a non-NULL pointer is passed (synchronises). */
typedef struct {
    int64_t insertions;      /* edges inserted by the call                          */
    int64_t case_count[3];   /* (root, insertion) scenarios in Case 1 / 2 / 3 */
    int64_t touched;         /* vertices touched (t[v] != untouched)       */
    int64_t down_vertices;   /* vertices whose sigma was recomputed (stage 2)        */
    int64_t edges_scanned;   /* adjacency entries read                               */
    int64_t alg_bytes;       /* algorithmic bytes of the update    */
} dbc_insert_stats;

typedef struct {
    float append_ms;   /* graph validation + append of the last insert call    */
    float update_ms;   /* update kernel(s) of the last insert call             */
    float static_ms;   /* last dbc_static_compute                              */
    int32_t update_launches;  /* update kernel launches in the last insert call */
    int32_t kernel_launches;  /* all library kernels launched by the last insert call */
    int64_t static_alg_bytes; /* algorithmic bytes of the last static compute   */
    /* cumulative since dbc_create / dbc_reset_timings: */
    double append_ms_total;
    double update_ms_total;
    int64_t update_launches_total;
    int64_t kernel_launches_total;
    int64_t insertions_total;
    int64_t alg_bytes_total;   /* update kernels' algorithmic bytes            */
    int32_t heavy_roots;       /* roots run on the wide heavy lane in the last insert call */
    int32_t reserved2;
} dbc_timings;

/* Fills *opt with defaults (device 0, rank 0, world 1, automatic sizes). */
void dbc_options_default(dbc_options *opt);

/* Fills *t with "automatic" for every field. */
void dbc_tuning_default(dbc_tuning *t);

/* Writes a fresh 128-byte ncclUniqueId to out (rank 0 of a multi-GPU job; the
 * caller distributes it to every rank's dbc_options.nccl_id).  NCCL is loaded
 * at run time (libnccl.so.2; the copy PyTorch loaded, if any).
 * Errors: DBC_EINVAL (out NULL), DBC_ENCCL (no NCCL, or NCCL failed). */
dbc_status dbc_nccl_unique_id(void *out);

/* Creates a context from an undirected graph in CSR form and a root set.
 *  n        number of vertices, >= 1
 *  row_ptr  host int64[n+1], row_ptr[0] = 0, non-decreasing
 *  col      host int32[row_ptr[n]]; the CSR must be symmetric, without self
 *           loops or duplicate entries (undirected).  The order
 *           of each row is the canonical adjacency order; inserted neighbours
 *           are appended after it in insertion order.
 *  roots    host int32[k], distinct, in range (the sampled sources)
 *  k        >= 0 (k = 0 gives BC = 0)
 *  opt      nullable (defaults)
 * Validates everything (O(m log) on the host) and uploads the CSR; keeps a
 * sorted host copy of the rows (4 bytes per entry + 8 per vertex) for the
 * host-side validation of dbc_insert_edges.  The per-root state is allocated
 * but undefined until dbc_static_compute.
 * Errors: DBC_EINVAL, DBC_ENOMEM, DBC_ECUDA. */
dbc_status dbc_create(dbc_ctx **out, int32_t n, const int64_t *row_ptr,
                      const int32_t *col, const int32_t *roots, int32_t k,
                      const dbc_options *opt);

/* Brandes over this rank's root shard (Alg. 1): resets and
 * recomputes d, sigma, delta of every local root and the BC partial on the
 * CURRENT graph (all inserted edges included).  Asynchronous on the stream. */
dbc_status dbc_static_compute(dbc_ctx *c);

/* Inserts count >= 0 undirected edges (u[i], v[i]) given in HOST memory, with
 * exactly the semantics of count sequential single-edge insertions (P:440,
 * "reinserted one at a time").  The whole batch is validated before anything
 * changes (self loop, range, already present, duplicate in batch ->
 * DBC_EEDGE; capacity -> DBC_ECAPACITY).  Requires a prior
 * dbc_static_compute (DBC_ESTATE).  Batches of up to 64 edges are validated on
 * the host against the context's host copy of the adjacency (caller ids: the
 * original rows sorted, plus the inserted and deleted edges), so the call does
 * not wait for the device: the append and the update are enqueued
 * asynchronously behind earlier work on the stream (it synchronises only with
 * DBC_FLAG_TIMING, on the previous call's events, or when stats is non-NULL).
 * Larger batches are validated on the device and the call synchronises once
 * after validation; the update itself is enqueued asynchronously.  stats:
 * nullable. */
dbc_status dbc_insert_edges(dbc_ctx *c, const int32_t *u, const int32_t *v,
                            int64_t count, dbc_insert_stats *stats);

/* Same as dbc_insert_edges with u, v in DEVICE memory (int32[count] each),
 * read in order after the work queued on the context stream.  Validated on the
 * device; synchronises once after validation (and copies the batch, through
 * pinned staging allocated on first use, to the host copy of the adjacency). */
dbc_status dbc_insert_edges_device(dbc_ctx *c, const int32_t *u_device,
                                   const int32_t *v_device, int64_t count,
                                   dbc_insert_stats *stats);

/* Deletes count >= 0 undirected edges (u[i], v[i]) given in HOST memory, with
 * the semantics of count sequential single-edge deletions (the decremental
 * counterpart of P:440; P:144 names deletion as the adjacent workload).  The
 * whole batch is validated first (range, self loop, duplicate pair within the
 * batch, edge not present -> DBC_EEDGE; nothing changes on error).  Each edge
 * leaves a tombstone in both adjacency rows (the rows keep the order of their
 * remaining entries -- the canonical order of DESIGN.md R5); a later
 * insertion of the same edge appends it again.  Per root the update follows
 * DESIGN.md R20: Case 1 if d(u) == d(v); if u_low keeps another predecessor
 * only sigma below it changes; else the affected vertices move down (or
 * become unreachable: d = DBC_INF, sigma = delta = 0).  Requires a prior
 * dbc_static_compute (DBC_ESTATE); not available with
 * DBC_FLAG_EDGE_PARALLEL (DBC_EINVAL).  stats: nullable, as for insertions
 * (case_count[2] counts deletions that moved a vertex). */
dbc_status dbc_delete_edges(dbc_ctx *c, const int32_t *u, const int32_t *v,
                            int64_t count, dbc_insert_stats *stats);

/* Same as dbc_delete_edges with u, v in DEVICE memory (copied to the host
 * for the batch checks). */
dbc_status dbc_delete_edges_device(dbc_ctx *c, const int32_t *u_device,
                                   const int32_t *v_device, int64_t count,
                                   dbc_insert_stats *stats);

/* Copies the GLOBAL BC (Eq. (3) over every root of every rank) to host
 * bc[n].  world == 1: this rank's sum.  world > 1: the per-rank partials are
 * summed by an all-reduce -- the context's NCCL communicator (opt.nccl_id) or
 * the opt.reduce callback; a collective call, every rank must make it.
 * Synchronises.  Errors: DBC_ESTATE (world > 1 without nccl_id or reduce; use
 * dbc_get_bc_partial_device), DBC_ENCCL (the reduction failed), DBC_ENUMERIC
 * (an earlier update overflowed). */
dbc_status dbc_get_bc(dbc_ctx *c, double *bc);

/* The same global BC left in DEVICE memory (fp64[n], caller's vertex order,
 * valid until the next call that returns a BC buffer, or destroy); the
 * all-reduce is enqueued on the context stream (a reduce callback may
 * synchronise).  A collective call at world > 1.  Errors as dbc_get_bc. */
dbc_status dbc_get_bc_device(dbc_ctx *c, double **bc_device);

/* Device pointer to this rank's BC partial, fp64[n] in the caller's vertex
 * order (a copy refreshed by this call, valid until the next call or destroy);
 * for a sum all-reduce across ranks.  Asynchronous on the context stream. */
dbc_status dbc_get_bc_partial_device(dbc_ctx *c, double **bc_device);

/* Copies one root's state to host arrays of n elements (any may be NULL).
 * slot: global slot in [0, k); must be owned by this rank (slot % world ==
 * rank), else DBC_EINVAL.  Synchronises. */
dbc_status dbc_get_root_state(dbc_ctx *c, int32_t slot, int32_t *d,
                              double *sigma, double *delta);

/* Number of root slots owned by this rank. */
dbc_status dbc_num_local_roots(const dbc_ctx *c, int32_t *k_local);

/* Waits for all enqueued work; reports deferred errors (DBC_ENUMERIC, DBC_ECUDA). */
dbc_status dbc_synchronize(dbc_ctx *c);

/* Kernel timings (CUDA events on the context stream; requires DBC_FLAG_TIMING)
 * of the last calls plus cumulative totals.  Synchronises. */
dbc_status dbc_get_timings(dbc_ctx *c, dbc_timings *t);

/* Zeroes the cumulative fields of dbc_timings.  Synchronises. */
dbc_status dbc_reset_timings(dbc_ctx *c);

/* Diagnostic counters (cumulative since create; layout is internal and may
 * change): case counts, touched, down vertices, scanned entries, algorithmic
 * bytes, static bytes, then scanned entries per update phase (down, removal,
 * down-vertex pull, down-vertex push, up vertices at level 2, at level >= 3).
 * Fills min(count, available) values.  Synchronises. */
dbc_status dbc_debug_counters(dbc_ctx *c, int64_t *out, int32_t count);

/* Diagnostic per-root profile of the update kernel: enable != 0 turns recording
 * on for later insert calls; out (nullable, int64[6 * k_local]) receives, per
 * local root slot of the last update launch, {start ns, end ns, working
 * (Case 2/3) insertions, touched vertices, adjacency entries scanned, level
 * steps}.  Synchronises when out != NULL. */
dbc_status dbc_debug_root_profile(dbc_ctx *c, int32_t enable, int64_t *out);

/* Diagnostic: per worker CTA of the last per-insertion (update_lean) launch run
 * with the root profile on, {entry, end of its root and help loops, exit}
 * globaltimer ns; worker w at out[3w..3w+2], 0 for a CTA that was not
 * launched.  *count receives the number of values (3 x scratch sets); out may
 * be NULL to query it; capacity < *count -> DBC_EINVAL.  Synchronises. */
dbc_status dbc_debug_cta_profile(dbc_ctx *c, int64_t *out, int64_t capacity, int64_t *count);

/* Scenario log (Fig. 2 and Fig. 4).  max_insertions > 0
 * turns it on for later insert calls whose batch has at most that many
 * insertions (larger batches -> DBC_EINVAL); while it is on, every (root,
 * insertion) is repaired as its own job (as with DBC_FLAG_NO_MERGE) so that
 * each scenario has its own record.  0 turns it off.  Allocates
 * 8 * max_insertions * k_local bytes of device memory. */
dbc_status dbc_scenario_log(dbc_ctx *c, int64_t max_insertions);

/* Copies the scenario log of the last insert call to host out[count]:
 * record [i * k_local + j] is insertion i of the batch seen by local root slot
 * j (local slot j = global slot j * world + rank), encoded as
 * case | (touched << 2) | (down << 33): case 1, 2 or 3;
 * touched = number of vertices the update touched, Alg. 2's
 * {v : t[v] != untouched} with the root excluded -- with the log on,
 * every DAG ancestor of a changed vertex is claimed even over a zero
 * Delta-delta push (R19); down = |D|, the vertices whose d/sigma were
 * recomputed.  Both 0 for Case 1.
 * *count receives the number of records; out may be NULL to query it.
 * capacity < *count -> DBC_EINVAL.  Synchronises. */
dbc_status dbc_get_scenarios(dbc_ctx *c, int64_t *out, int64_t capacity, int64_t *count);

/* Device memory held by the context, in bytes. */
dbc_status dbc_device_bytes(const dbc_ctx *c, int64_t *bytes);

const char *dbc_strerror(dbc_status s);
const char *dbc_last_error(const dbc_ctx *c);
int32_t dbc_abi_version(void);

/* Frees everything; NULL is a no-op. */
void dbc_destroy(dbc_ctx *c);

#ifdef __cplusplus
}
#endif
#endif /* DBC_H */
